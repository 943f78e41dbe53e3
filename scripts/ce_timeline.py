"""Experiment: timeline of copy-engine migrations (kernel = 3) next to the decode victim —
do they overlap, and at what rate?  Development tool."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
import victim  # noqa: E402
from windgen import migration_case, SHAPES  # noqa: E402

dev = torch.device("cuda", 0)
sh = SHAPES["C3"]
B, ctx_len, bs = 16, 2048, 16
nbv = B * ctx_len // bs
vpool = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, 2, nbv)
vt = vpool.tensor().view(torch.float16)
for o in range(0, vt.numel(), 1 << 28):
    vt[o:o + (1 << 28)].normal_()
bt = torch.randperm(nbv).to(torch.int32).view(B, -1).to(dev)
ctx = torch.full((B,), ctx_len, dtype=torch.int32, device=dev)
q = torch.randn(B, sh.n_kv_heads, 128, device=dev, dtype=torch.float16)
scratch = torch.empty(victim.scratch_floats(B, sh.n_kv_heads, ctx_len // bs, 64), device=dev)
out = torch.empty(B, sh.n_kv_heads, 128, device=dev)
plane = nbv * sh.chunk_bytes
hi_s = torch.cuda.Stream(0, priority=-1)
lo_s = torch.cuda.Stream(0, priority=0)
case = migration_case("C3")
src = bench.make_pool(wk, sh, case.nb_src, 0, 1, 1)
dst = bench.make_pool(wk, sh, case.nb_dst, 0, 1, 2)
hs, hd = torch.as_tensor(case.src_bt).pin_memory(), torch.as_tensor(case.dst_bt).pin_memory()
pb = bench.payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
RATE = int(sys.argv[1]) if len(sys.argv) > 1 else 0
wk.set_tuning(wk.PATH_INTRA, kernel=wk.KERNEL_COPY_ENGINE, rate_mbps=RATE * 1000)


def victim_steps(n):
    for _ in range(n):
        for l in range(sh.n_layers):
            kp = vpool.base + 2 * l * plane
            victim.decode_attention(q, kp, kp + plane, bt, ctx, sh.n_kv_heads, bs, scratch, out,
                                    blocks_per_split=64, stream=hi_s.cuda_stream)


victim_steps(3)
torch.cuda.synchronize()
res = {}
for mode in ("ce_alone", "victim_alone", "both"):
    t0 = torch.cuda.Event(enable_timing=True)
    t0.record(lo_s)
    hi_s.wait_stream(lo_s)
    ce_ev, v_ev = [], []
    n_mig = 20 if mode != "victim_alone" else 0
    n_vic = 20 if mode != "ce_alone" else 0
    for i in range(max(n_mig, n_vic)):
        if i < n_mig:
            wk.migrate(src, hs.data_ptr(), dst, hd.data_ptr(), n=case.n, stream=lo_s)
            e = torch.cuda.Event(enable_timing=True)
            e.record(lo_s)
            ce_ev.append(e)
        if i < n_vic:
            victim_steps(1)
            e = torch.cuda.Event(enable_timing=True)
            e.record(hi_s)
            v_ev.append(e)
    torch.cuda.synchronize()
    r = {}
    if ce_ev:
        r["ce_end_ms"] = [round(t0.elapsed_time(e), 2) for e in ce_ev[::4]]
        r["ce_gbs"] = round(pb * n_mig / t0.elapsed_time(ce_ev[-1]) / 1e6, 1)
    if v_ev:
        r["victim_end_ms"] = [round(t0.elapsed_time(e), 2) for e in v_ev[::4]]
        r["victim_step_ms"] = round(t0.elapsed_time(v_ev[-1]) / n_vic, 3)
    res[mode] = r
print(json.dumps(res))
