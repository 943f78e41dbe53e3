"""ncu target: fixed per-op cost — 1-block and 8-block C1 migrates (12 layers), and the same
through the SIMT kernel."""
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
a = bench.make_pool(wk, sh, case.nb_src, 0, case.content_seed, case.src_tag)
b = bench.make_pool(wk, sh, case.nb_dst, 0, case.content_seed, case.dst_tag)
sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
for n in (1, 1, 8, case.n):
    wk.migrate(a, sbt[:n], b, dbt[:n])
torch.cuda.synchronize()
