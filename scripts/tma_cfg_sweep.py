"""Development helper: full-size migrate of one config under explicit TMA / SIMT tunings
(CUDA events, back-to-back, inputs >> L2)."""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
from windgen import migration_case  # noqa: E402

cfg = sys.argv[1]
dev = torch.device("cuda", 0)
case = migration_case(cfg, scale=float(sys.argv[2]) if len(sys.argv) > 2 else 1.0)
sh = case.shape
a = bench.make_pool(wk, sh, case.nb_src, 0, case.content_seed, case.src_tag)
b = bench.make_pool(wk, sh, case.nb_dst, 0, case.content_seed, case.dst_tag)
sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
s = torch.cuda.Stream(dev)
pb = bench.payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
T, S = wk.KERNEL_TMA, wk.KERNEL_SIMT
out = {}
for name, t in [("default", None),
                ("t32k_s6_l3", wk.tuning(kernel=T, stage_bytes=32768, stages=6, store_lag=3)),
                ("t32k_s6_l2", wk.tuning(kernel=T, stage_bytes=32768, stages=6, store_lag=2)),
                ("t32k_s6_l4", wk.tuning(kernel=T, stage_bytes=32768, stages=6, store_lag=4)),
                ("t64k_s3_l1", wk.tuning(kernel=T, stage_bytes=65536, stages=3, store_lag=1)),
                ("t32k_s3_l1_2cta", wk.tuning(kernel=T, stage_bytes=32768, stages=3, store_lag=1, ctas_per_sm=2)),
                ("t16k_s12_l6", wk.tuning(kernel=T, stage_bytes=16384, stages=12, store_lag=6)),
                ("t48k_s4_l2", wk.tuning(kernel=T, stage_bytes=49152, stages=4, store_lag=2)),
                ("simt_4cta_32k", wk.tuning(kernel=S, stage_bytes=32768, stages=4, ctas_per_sm=4))]:
    ms = bench.time_device(lambda: wk.migrate_ex(a, sbt, b, dbt, t, stream=s), 5, 3, s) / 5
    out[name] = round(pb / ms / 1e6, 1)
    print(cfg, name, out[name], round(2 * out[name] / 6550, 3), flush=True)
print(json.dumps({cfg: out}))
