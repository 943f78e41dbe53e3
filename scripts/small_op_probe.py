"""Development probe (round 2): where the fixed cost of a small op goes.  The C1 intra-device
migrate (144 MiB) and the C1 compaction (67 moves, 39.5 MB), each timed alone between two
CUDA events after an L2 flush (as bench.py's c1_intra), under several tunings; plus a
'floor': the same event pair around an empty kernel, and around a 1-block op.
Usage: python scripts/small_op_probe.py [--ncu]   (--ncu: 3 reps, for a launch list)"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
from windgen import migration_case, live_mask_after_free, request_lengths, blocks_for_tokens  # noqa: E402

dev = torch.device("cuda", 0)
REPS = 3 if "--ncu" in sys.argv else 30
case = migration_case("C1")
sh = case.shape
a = bench.make_pool(wk, sh, case.nb_src, 0, case.content_seed, case.src_tag)
b = bench.make_pool(wk, sh, case.nb_dst, 0, case.content_seed, case.dst_tag)
sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
reqb = blocks_for_tokens(request_lengths("C1"), sh.block_size)
live, _ = live_mask_after_free(case.nb_src, reqb, 0.5, 4001)
csrc, cdst = wk.plan_compact(live)
ts, td = torch.as_tensor(csrc, device=dev), torch.as_tensor(cdst, device=dev)
flush = torch.ones(2 * (126 << 20) // 4, dtype=torch.int32, device=dev)
s = torch.cuda.Stream(dev)
pb = bench.payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
pc = bench.payload_bytes(len(csrc), sh.n_layers, sh.chunk_bytes)
hbm = json.load(open("MEASURED_PEAKS.json"))["hbm_gbs"] if os.path.exists("MEASURED_PEAKS.json") else 6650.0
tiny = torch.zeros(1, device=dev)


def timed(fn, reps=REPS, do_flush=True):
    for _ in range(3):
        fn()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        for e0, e1 in ev:
            if do_flush:
                flush.sum(dtype=torch.int64)
            e0.record(s)
            fn()
            e1.record(s)
    torch.cuda.synchronize()
    return float(np.median([e0.elapsed_time(e1) for e0, e1 in ev])) * 1e3  # us


out = {"hbm_gbs": hbm, "ideal_us_migrate": round(2 * pb / hbm / 1e3, 2),
       "ideal_us_compact": round(2 * pc / hbm / 1e3, 2), "moves": int(len(csrc))}
out["floor_empty_kernel_us"] = round(timed(lambda: tiny.add_(0)), 2)
print("floor (event pair around a 1-thread torch kernel after the flush):", out["floor_empty_kernel_us"], "us", flush=True)
T, S = wk.KERNEL_TMA, wk.KERNEL_SIMT
tunings = [("default", None),
           ("tma_u48k_s4_2cta", wk.tuning(kernel=T, stage_bytes=49152, stages=4, store_lag=2, ctas_per_sm=2)),
           ("tma_u24k_s4", wk.tuning(kernel=T, stage_bytes=24576, stages=4, store_lag=2)),
           ("tma_u24k_s6_2cta", wk.tuning(kernel=T, stage_bytes=24576, stages=6, store_lag=3, ctas_per_sm=2)),
           ("tma_u24k_s3_3cta", wk.tuning(kernel=T, stage_bytes=24576, stages=3, store_lag=1, ctas_per_sm=3)),
           ("simt_u24k_2cta", wk.tuning(kernel=S, stage_bytes=24576, stages=4, ctas_per_sm=2)),
           ("simt_u24k_4cta", wk.tuning(kernel=S, stage_bytes=24576, stages=4, ctas_per_sm=4)),
           ("simt_u48k_4cta", wk.tuning(kernel=S, stage_bytes=49152, stages=4, ctas_per_sm=4))]
if "--ring" in sys.argv:  # bytes in flight per CTA for small ops (stage x stages, store lag)
    tunings = [("default", None)] + [
        (f"tma_u{sb // 1024}k_s{st}_lag{lag}", wk.tuning(kernel=T, stage_bytes=sb, stages=st, store_lag=lag))
        for sb, st, lag in ((49152, 4, 1), (49152, 4, 3), (32768, 6, 2), (32768, 6, 1),
                            (24576, 8, 2), (24576, 8, 1), (16384, 12, 3), (16384, 12, 2), (12288, 16, 4))]
for name, t in tunings:
    r = {}
    for op, fn, by in (("migrate", lambda: wk.migrate_ex(a, sbt, b, dbt, t, stream=s), pb),
                       ("compact", lambda: wk.migrate_ex(a, ts, a, td, t, stream=s), pc),
                       ("one_block", lambda: wk.migrate_ex(a, sbt[:1], b, dbt[:1], t, stream=s), 0)):
        try:
            us = timed(fn)
        except wk.WindKVError as e:
            print(name, op, "failed:", e, None if t is None else [(f, getattr(t, f)) for f, _ in t._fields_])
            continue
        r[op + "_us"] = round(us, 2)
        if by:
            r[op + "_frac"] = round(2 * by / (us * 1e-6) / 1e9 / hbm, 3)
    # back to back (no flush, no event between): the per-op cost in a stream of ops
    if len(r) < 5:
        continue
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    with torch.cuda.stream(s):
        ev0.record(s)
        for _ in range(20):
            wk.migrate_ex(a, ts, a, td, t, stream=s)
        ev1.record(s)
    torch.cuda.synchronize()
    r["compact_b2b_us"] = round(ev0.elapsed_time(ev1) / 20 * 1e3, 2)
    out[name] = r
    print(name, r, flush=True)
print(json.dumps(out))
