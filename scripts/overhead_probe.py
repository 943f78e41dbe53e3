"""Where does a short op lose time?  (development probe, one B200; not the bench)

C5 geometry (fp8, C = 16 KiB).  Times, on one stream with CUDA events:
  * the C5 compaction (same pool) and the same (src, dst) pairs between two pools;
  * shuffled and sequential tables of the same size;
  * sequential ops of growing size, to fit time = fixed + bytes / rate.
"""
import json
import math
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
import windgen.cuda as wg  # noqa: E402
from windgen import SHAPES, request_lengths, skewed_placement, blocks_for_tokens, live_mask_after_free  # noqa: E402

PEAK = bench.load_peaks()["hbm_gbs"]
dev = torch.device("cuda", 0)
s = torch.cuda.Stream(dev)
sh = SHAPES["C5"]


def pool(nb, tag):
    p = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nb)
    wg.fill(p.base, p.nbytes, 0, 1, tag)
    return p


def timeit(fn, reps=20, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    for _ in range(reps):
        fn()
    b.record(s)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def rep(name, n, ms, **kw):
    pb = 2 * sh.n_layers * n * sh.chunk_bytes
    print(json.dumps(dict(probe=name, n=n, ms=round(ms, 4), gbs=round(pb / ms / 1e6, 1),
                          frac=round(2 * pb / ms / 1e6 / PEAK, 4), **kw)), flush=True)


lens = request_lengths("C5")
place = skewed_placement(lens.size, 8, 4005)
reqb = blocks_for_tokens(lens[place == 0], 16)
nb = math.ceil(int(reqb.sum()) * 1.1)
live, _ = live_mask_after_free(nb, reqb, 0.5, 4006)
cs, cd = wk.plan_compact(live)
n = len(cs)
A, B = pool(nb, 1), pool(nb, 2)
tcs, tcd = torch.as_tensor(cs, device=dev), torch.as_tensor(cd, device=dev)
rep("compact_same_pool", n, timeit(lambda: wk.compact(A, tcs, tcd, stream=s)))
rep("compact_pairs_two_pools", n, timeit(lambda: wk.migrate(A, tcs, B, tcd, stream=s)))
rng = np.random.default_rng(0)
perm = torch.as_tensor(rng.permutation(nb)[:n].astype(np.int32), device=dev)
perm2 = torch.as_tensor(rng.permutation(nb)[:n].astype(np.int32), device=dev)
rep("shuffled_both", n, timeit(lambda: wk.migrate(A, perm, B, perm2, stream=s)))
seq = torch.arange(n, dtype=torch.int32, device=dev)
rep("sequential", n, timeit(lambda: wk.migrate(A, seq, B, seq, stream=s)))
for m in (256, 1024, 2048, 4096, 8192, 14000):
    t = torch.arange(m, dtype=torch.int32, device=dev)
    rep("sequential_size", m, timeit(lambda: wk.migrate(A, t, B, t, stream=s)))
    tp = torch.as_tensor(rng.permutation(nb)[:m].astype(np.int32), device=dev)
    rep("shuffled_size", m, timeit(lambda: wk.migrate(A, tp, B, t, stream=s)))
# empty-ish op: one block, all layers (launch + ramp + publish)
one = torch.zeros(1, dtype=torch.int32, device=dev)
rep("one_block", 1, timeit(lambda: wk.migrate(A, one, B, one, stream=s), reps=200))
# back-to-back split: the compaction as 4 ops of n/4 pairs
q = n // 4
parts = [(tcs[i * q:(i + 1) * q if i < 3 else n], tcd[i * q:(i + 1) * q if i < 3 else n]) for i in range(4)]


def four():
    for a, b in parts:
        wk.compact(A, a, b, stream=s)
rep("compact_as_4_ops", n, timeit(four))
rep("one_block_one_layer", 1, timeit(lambda: wk.migrate(A, one, B, one, layer_lo=0, layer_hi=1, stream=s), reps=200))
rep("one_block_8_layers", 1, timeit(lambda: wk.migrate(A, one, B, one, layer_lo=0, layer_hi=8, stream=s), reps=200))
