"""Experiment: interference of a copy-engine (DMA, zero SMs) migration with the HBM-bound
decode victim, vs the SM kernels at a similar rate.  Development tool."""
import json
import math
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


def victim_run(n):
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(n + 1)]
    ev[0].record(hi_s)
    for i in range(n):
        for l in range(sh.n_layers):
            kp = vpool.base + 2 * l * plane
            victim.decode_attention(q, kp, kp + plane, bt, ctx, sh.n_kv_heads, bs, scratch, out,
                                    blocks_per_split=64, stream=hi_s.cuda_stream)
        ev[i + 1].record(hi_s)
    torch.cuda.synchronize()
    return float(np.median([ev[i].elapsed_time(ev[i + 1]) for i in range(n)]))


case = migration_case("C3")
src = bench.make_pool(wk, sh, case.nb_src, 0, 1, 1)
dst = bench.make_pool(wk, sh, case.nb_dst, 0, 1, 2)
pb = bench.payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
planes = 2 * sh.n_layers
victim_run(5)


def ce_once():
    victim.ce_gather("loop", src.base, case.nb_src * sh.chunk_bytes, dst.base, case.nb_dst * sh.chunk_bytes,
                     sh.chunk_bytes, case.src_bt, case.dst_bt, planes, lo_s.cuda_stream)


t_ce = bench.time_device(ce_once, 1, 1, lo_s)
res = {"ce_gbs_alone": round(pb / t_ce / 1e6, 1)}
import threading  # noqa: E402
import time  # noqa: E402

for rnd in range(3):
    a = victim_run(20)
    stop = threading.Event()
    done = []

    def feeder():  # keeps the copy engines busy while the victim runs (ctypes drops the GIL)
        while not stop.is_set():
            ce_once()
            done.append(1)
    th = threading.Thread(target=feeder)
    th.start()
    time.sleep(0.3)
    e0 = torch.cuda.Event(enable_timing=True)
    e0.record(lo_s)
    w = victim_run(20)
    stop.set()
    th.join()
    e1 = torch.cuda.Event(enable_timing=True)
    e1.record(lo_s)
    torch.cuda.synchronize()
    res[f"round{rnd}"] = {"alone": round(a, 3), "with_ce": round(w, 3), "slowdown": round(w / a - 1, 4),
                          "ce_ops_enqueued": len(done), "ce_stream_span_ms": round(e0.elapsed_time(e1), 1)}
print(json.dumps(res))
