"""Small driver for ncu captures of the secondary kernels: the SIMT copy kernel on a
C2-shaped migration and the victim decode-attention split kernel."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
import victim  # noqa: E402
import windgen.cuda as wg  # noqa: E402
from windgen import migration_case, SHAPES  # noqa: E402

dev = torch.device("cuda", 0)
case = migration_case("C2", scale=0.25)
sh = case.shape
src = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, case.nb_src)
dst = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, case.nb_dst)
wg.fill(src.base, src.nbytes, 0, 1, 1)
sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
wk.set_tuning(wk.PATH_INTRA, kernel=wk.KERNEL_SIMT, ctas_per_sm=4, stage_bytes=131072, stages=6)
for _ in range(3):
    wk.migrate(src, sbt, dst, dbt)
torch.cuda.synchronize()
print("simt payload bytes per launch", 2 * sh.n_layers * case.n * sh.chunk_bytes)
del src, dst
sh3 = SHAPES["C3"]
B, T = 16, 2048
nb = B * T // 16
vp = wk.Pool(4, sh3.n_kv_heads, 128, 16, 2, nb)
vp.tensor().view(torch.float16).normal_()
bt = torch.randperm(nb).to(torch.int32).view(B, -1).to(dev)
ctx = torch.full((B,), T, dtype=torch.int32, device=dev)
q = torch.randn(B, sh3.n_kv_heads, 128, device=dev, dtype=torch.float16)
scratch = torch.empty(victim.scratch_floats(B, sh3.n_kv_heads, T // 16, 64), device=dev)
out = torch.empty(B, sh3.n_kv_heads, 128, device=dev)
plane = nb * sh3.chunk_bytes
for l in range(4):
    victim.decode_attention(q, vp.base + 2 * l * plane, vp.base + (2 * l + 1) * plane, bt, ctx,
                            sh3.n_kv_heads, 16, scratch, out, blocks_per_split=64)
torch.cuda.synchronize()
print("victim kv bytes per launch", 2 * B * T * sh3.n_kv_heads * 128 * 2)
