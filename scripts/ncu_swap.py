"""ncu target: C1 host swaps through the SM kernel on mapped pinned memory (swap-out at the
default ~384 KiB in flight and at 8 CTAs, swap-in at 8 CTAs) and one staged swap-out
(its gather kernels are intra-device; the PCIe bytes move by DMA, outside any kernel)."""
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
src = bench.make_pool(wk, sh, case.nb_src, 0, case.content_seed, case.src_tag)
host = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, case.n, loc="host")
sbt = torch.as_tensor(case.src_bt, device=dev)
hd = torch.arange(case.n, dtype=torch.int32, device=dev)
hh = torch.arange(case.n, dtype=torch.int32).pin_memory()
saved = wk.get_tuning(wk.PATH_HOST)
wk.set_tuning(wk.PATH_HOST, **{**saved, "kernel": wk.KERNEL_TMA})
wk.swap_out(src, sbt, host, hd)                       # launch 1: SM swap-out, default grid
wk.set_tuning(wk.PATH_HOST, **{**saved, "kernel": wk.KERNEL_TMA, "max_ctas": 8})
wk.swap_out(src, sbt, host, hd)                       # launch 2: SM swap-out, 8 CTAs
wk.set_tuning(wk.PATH_HOST, **{**saved, "kernel": wk.KERNEL_TMA})
wk.swap_in(host, hd, src, sbt)                        # launch 3: SM swap-in, 8 CTAs
wk.set_tuning(wk.PATH_HOST, **saved)
wk.swap_out(src, sbt, host, hh)                       # launches 4..: staged gathers
torch.cuda.synchronize()
print("payload bytes per swap", bench.payload_bytes(case.n, sh.n_layers, sh.chunk_bytes))
