"""Development probe: C1 swap_out / swap_in on the default HOST path (bench c1_swap), GB/s,
to A/B library builds (run from each build's tree).  Usage: python scripts/swap_ab.py <label>"""
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
from windgen import migration_case  # noqa: E402

dev = torch.device("cuda", 0)
case = migration_case("C1")
sh = case.shape
dpool = bench.make_pool(wk, sh, case.nb_src, 0, case.content_seed, case.src_tag)
dpool2 = bench.make_pool(wk, sh, case.nb_dst, 0, case.content_seed, case.dst_tag)
hpool = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, case.n, loc="host")
hbt = torch.arange(case.n, dtype=torch.int32, device=dev)
sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
pb = bench.payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
s = torch.cuda.Stream(dev)
r = {"label": sys.argv[1] if len(sys.argv) > 1 else ""}
for rep in range(2):
    ms_o = bench.time_device(lambda: wk.swap_out(dpool, sbt, hpool, hbt, stream=s), 10, 3, s) / 10
    ms_i = bench.time_device(lambda: wk.swap_in(hpool, hbt, dpool2, dbt, stream=s), 10, 3, s) / 10
    r[f"out_gbs_{rep}"] = round(pb / ms_o / 1e6, 2)
    r[f"in_gbs_{rep}"] = round(pb / ms_i / 1e6, 2)
print(json.dumps(r), flush=True)
