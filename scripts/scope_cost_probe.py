"""Development probe (round 2): the cost of system-scope layer publication (what every peer /
NVLink destination needs) against GPU scope, on one GPU.  Run twice — with and without
WIND_KV_FORCE_SYS_SCOPE=1 — and compare: a 1-block op and a 16-block op over all 40 layers of
the C2 geometry (publication-dominated), the full C2 migrate, and the 40-launch
layer-streamed C2 hand-off.  Back to back on one stream (no flush), CUDA events."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
from windgen import migration_case  # noqa: E402

dev = torch.device("cuda", 0)
case = migration_case("C2")
sh = case.shape
src = bench.make_pool(wk, sh, case.nb_src, 0, case.content_seed, case.src_tag)
dst = bench.make_pool(wk, sh, case.nb_dst, 0, case.content_seed, case.dst_tag)
sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
s, cons = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
_, _, scope = wk.route(src, dst)
out = {"sys_scope": scope}
for n in (1, 16):
    ms = bench.time_device(lambda: wk.migrate(src, sbt[:n], dst, dbt[:n], stream=s), 50, 5, s) / 50
    out[f"op_{n}_blocks_40_layers_us"] = round(ms * 1e3, 2)
pb = bench.payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
ms = bench.time_device(lambda: wk.migrate(src, sbt, dst, dbt, stream=s), 5, 2, s) / 5
out["c2_full_gbs"] = round(pb / ms / 1e6, 1)


def streamed():
    for l in range(sh.n_layers):
        wk.migrate(src, sbt, dst, dbt, layer_lo=l, layer_hi=l + 1, stream=s)
    t = dst.layer_ticket()
    for l in range(sh.n_layers):
        wk.layer_wait(dst, l, t, stream=cons)
    s.wait_stream(cons)


ms = bench.time_device(streamed, 5, 2, s) / 5
out["c2_layer_streamed_gbs"] = round(pb / ms / 1e6, 1)
print(json.dumps(out))
