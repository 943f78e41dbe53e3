"""Tuning sweep for the copy kernels on one B200 (development tool, not the bench).

Prints one JSON line per configuration: payload GB/s and DRAM fraction of the measured
copy peak for the C2 (160 KiB chunks) and C5 (16 KiB chunks) shapes, shuffled tables.
"""
import json
import math
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
import windgen.cuda as wg  # noqa: E402
from windgen import migration_case, SHAPES, KVShape  # noqa: E402

import bench  # noqa: E402

PEAK = bench.load_peaks()["hbm_gbs"]
dev = torch.device("cuda", 0)


def pool(sh, nb, tag):
    p = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nb)
    wg.fill(p.base, p.nbytes, 0, 1, tag)
    return p


def timeit(fn, stream, reps=10, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(stream)
    for _ in range(reps):
        fn()
    b.record(stream)
    torch.cuda.synchronize()
    return a.elapsed_time(b) / reps


def host_sweep():
    """Host swap path: C1 and C4 geometries, swap_out / swap_in, kernel x CTAs x unit."""
    s = torch.cuda.Stream(dev)
    for name, sh, nblk in [("C1", SHAPES["C1"], 256), ("C4", SHAPES["C4"], 512)]:
        dpool = pool(sh, nblk + 10, 1)
        hpool = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes,
                        nblk, loc="host")
        bt = torch.randperm(nblk + 10)[:nblk].to(torch.int32).to(dev)
        hbt = torch.arange(nblk, dtype=torch.int32, device=dev)
        bt_h, hbt_h = bt.cpu().pin_memory(), hbt.cpu().pin_memory()
        pb = 2 * sh.n_layers * nblk * sh.chunk_bytes
        for cfg in [dict(kernel=wk.KERNEL_SIMT, ctas_per_sm=4, stage_bytes=32768),
                    dict(kernel=wk.KERNEL_SIMT, ctas_per_sm=2, stage_bytes=32768),
                    dict(kernel=wk.KERNEL_SIMT, ctas_per_sm=1, stage_bytes=65536),
                    dict(kernel=wk.KERNEL_SIMT, ctas_per_sm=4, stage_bytes=131072),
                    dict(kernel=wk.KERNEL_TMA, ctas_per_sm=1, stage_bytes=49152, stages=4),
                    dict(kernel=wk.KERNEL_TMA, ctas_per_sm=1, stage_bytes=32768, stages=6),
                    dict(kernel=wk.KERNEL_TMA, ctas_per_sm=2, stage_bytes=16384, stages=6),
                    dict(kernel=wk.KERNEL_SIMT, ctas_per_sm=4, stage_bytes=32768, max_ctas=64),
                    dict(kernel=wk.KERNEL_TMA, ctas_per_sm=1, stage_bytes=49152, stages=4, max_ctas=64),
                    dict(kernel=wk.KERNEL_TMA, ctas_per_sm=1, stage_bytes=49152, stages=4, max_ctas=32),
                    dict(kernel=wk.KERNEL_TMA, ctas_per_sm=1, stage_bytes=49152, stages=4, max_ctas=16),
                    dict(kernel=wk.KERNEL_TMA, ctas_per_sm=1, stage_bytes=49152, stages=4, max_ctas=8),
                    dict(kernel=wk.KERNEL_TMA, ctas_per_sm=1, stage_bytes=49152, stages=4, max_ctas=4),
                    dict(kernel=wk.KERNEL_TMA, ctas_per_sm=1, stage_bytes=32768, stages=6, max_ctas=8),
                    dict(kernel=wk.KERNEL_SIMT, ctas_per_sm=1, stage_bytes=65536, max_ctas=8),
                    dict(kernel=wk.KERNEL_COPY_ENGINE, stage_bytes=49152, stages=4)]:
            wk.set_tuning(wk.PATH_HOST, **cfg)
            ce = cfg["kernel"] == wk.KERNEL_COPY_ENGINE
            a, b = (bt_h, hbt_h) if ce else (bt, hbt)
            mo = timeit(lambda: wk.swap_out(dpool, a, hpool, b, n=nblk, stream=s), s, reps=5)
            mi = timeit(lambda: wk.swap_in(hpool, b, dpool, a, n=nblk, stream=s), s, reps=5)
            print(json.dumps(dict(case=name, mode="host", **cfg, out_gbs=round(pb / mo / 1e6, 2),
                                  in_gbs=round(pb / mi / 1e6, 2))), flush=True)
        hb = torch.empty(pb, dtype=torch.uint8, pin_memory=True)
        db = torch.empty(pb, dtype=torch.uint8, device=dev)
        cs = torch.cuda.current_stream(dev)
        d2h = timeit(lambda: hb.copy_(db, non_blocking=True), cs, reps=5)
        h2d = timeit(lambda: db.copy_(hb, non_blocking=True), cs, reps=5)
        print(json.dumps(dict(case=name, mode="copy_engine", d2h_gbs=round(pb / d2h / 1e6, 2),
                              h2d_gbs=round(pb / h2d / 1e6, 2))), flush=True)
        del dpool, hpool


def victim_check():
    import victim
    from windgen import SHAPES as SH
    sh = SH["C3"]
    B, ctx_len, bs = 16, 2048, 16
    nbv = B * ctx_len // bs
    vp = wk.Pool(8, sh.n_kv_heads, sh.head_dim, bs, 2, nbv)
    vt = vp.tensor().view(torch.float16)
    vt.normal_()
    bt = torch.randperm(nbv).to(torch.int32).view(B, -1).to(dev)
    ctx = torch.full((B,), ctx_len, dtype=torch.int32, device=dev)
    q = torch.randn(B, sh.n_kv_heads, 128, device=dev, dtype=torch.float16)
    plane = nbv * sh.chunk_bytes
    for bps in (16, 32, 64):
        scratch = torch.empty(victim.scratch_floats(B, sh.n_kv_heads, ctx_len // bs, bps), device=dev)
        out = torch.empty(B, sh.n_kv_heads, 128, device=dev)
        s = torch.cuda.current_stream(dev)

        def step():
            for l in range(8):
                kp = vp.base + 2 * l * plane
                victim.decode_attention(q, kp, kp + plane, bt, ctx, sh.n_kv_heads, bs, scratch, out,
                                        blocks_per_split=bps, stream=s.cuda_stream)
        ms = timeit(step, s, reps=10)
        kv = 8 * 2 * B * ctx_len * sh.n_kv_heads * 128 * 2
        print(json.dumps(dict(mode="victim", blocks_per_split=bps, ms=round(ms, 3),
                              hbm_frac=round(kv / ms / 1e6 / PEAK, 3))), flush=True)


def compact_sweep():
    """C5 compaction (same pool, fp8, C = 16 KiB) over TMA / SIMT configurations."""
    from windgen import request_lengths, skewed_placement, blocks_for_tokens, live_mask_after_free
    sh5 = SHAPES["C5"]
    lens = request_lengths("C5")
    place = skewed_placement(lens.size, 8, 4005)
    reqb = blocks_for_tokens(lens[place == 0], 16)
    nb = math.ceil(int(reqb.sum()) * 1.1)
    live, _ = live_mask_after_free(nb, reqb, 0.5, 4006)
    cs, cd = wk.plan_compact(live)
    runs = 1 + int(np.sum((np.diff(cs) != 1) | (np.diff(cd) != 1)))
    p = pool(sh5, nb, 1)
    ts, td = torch.as_tensor(cs, device=dev), torch.as_tensor(cd, device=dev)
    pb = 2 * sh5.n_layers * len(cs) * sh5.chunk_bytes
    s = torch.cuda.Stream(dev)
    print(json.dumps(dict(mode="compact_info", moves=len(cs), runs=runs, pool_blocks=nb)), flush=True)
    for cfg in [dict(kernel=wk.KERNEL_TMA, stage_bytes=49152, stages=4, ctas_per_sm=1, store_lag=2),
                dict(kernel=wk.KERNEL_TMA, stage_bytes=32768, stages=6, ctas_per_sm=1, store_lag=3),
                dict(kernel=wk.KERNEL_TMA, stage_bytes=32768, stages=6, ctas_per_sm=1, store_lag=2),
                dict(kernel=wk.KERNEL_TMA, stage_bytes=16384, stages=6, ctas_per_sm=2, store_lag=3),
                dict(kernel=wk.KERNEL_TMA, stage_bytes=16384, stages=12, ctas_per_sm=1, store_lag=6),
                dict(kernel=wk.KERNEL_TMA, stage_bytes=65536, stages=3, ctas_per_sm=1, store_lag=1),
                dict(kernel=wk.KERNEL_SIMT, stage_bytes=32768, ctas_per_sm=4),
                dict(kernel=wk.KERNEL_SIMT, stage_bytes=65536, ctas_per_sm=2)]:
        wk.set_tuning(wk.PATH_INTRA, **cfg)
        ms = timeit(lambda: wk.compact(p, ts, td, stream=s), s, reps=10)
        gbs = pb / ms / 1e6
        print(json.dumps(dict(case="C5compact", **cfg, ms=round(ms, 3), gbs=round(gbs, 1),
                              frac=round(2 * gbs / PEAK, 4))), flush=True)


def fanout_sweep():
    """Read-once fan-out (2 and 3 destinations, C2 geometry, half size) over TMA ring shapes."""
    sh = SHAPES["C2"]
    case = migration_case("C2", scale=0.5)
    src = pool(sh, case.nb_src, 1)
    dsts = [pool(sh, case.nb_dst, 2 + j) for j in range(3)]
    sbt = torch.as_tensor(case.src_bt, device=dev)
    dbt = torch.as_tensor(case.dst_bt, device=dev)
    pb = 2 * sh.n_layers * case.n * sh.chunk_bytes
    s = torch.cuda.Stream(dev)
    for k in (2, 3):
        for stage, stages, lag in [(49152, 4, 2), (49152, 4, 1), (49152, 4, 3), (32768, 6, 3), (32768, 6, 2),
                                   (32768, 6, 4), (24576, 8, 4), (40960, 5, 2), (65536, 3, 1)]:
            wk.set_tuning(wk.PATH_INTRA, kernel=wk.KERNEL_TMA, stage_bytes=stage, stages=stages, store_lag=lag,
                          ctas_per_sm=1)
            ms = timeit(lambda: wk.migrate_batch(src, [(d, sbt, dbt) for d in dsts[:k]], 0, sh.n_layers,
                                                 stream=s), s, reps=8)
            dram = (1 + k) * pb
            print(json.dumps(dict(case="fanout", k=k, stage_bytes=stage, stages=stages, store_lag=lag,
                                  ms=round(ms, 3), frac=round(dram / ms / 1e6 / PEAK, 4))), flush=True)


def main():
    which = sys.argv[1] if len(sys.argv) > 1 else "all"
    if which == "fanout":
        return fanout_sweep()
    if which == "host":
        return host_sweep()
    if which == "compact":
        return compact_sweep()
    if which == "victim":
        return victim_check()
    s = torch.cuda.Stream(dev)
    out = []
    cases = {}
    c2 = migration_case("C2")
    cases["C2"] = (c2.shape, c2)
    # C5-shaped (16 KiB chunks) with a similar ~20 GiB payload
    sh5 = SHAPES["C5"]
    c5 = migration_case("C5", shape=sh5, lengths=np.full(640, 1024))
    cases["C5"] = (sh5, c5)
    for name, (sh, case) in cases.items():
        src = pool(sh, case.nb_src, 1)
        dst = pool(sh, case.nb_dst, 2)
        sbt = torch.as_tensor(case.src_bt, device=dev)
        dbt = torch.as_tensor(case.dst_bt, device=dev)
        pb = 2 * sh.n_layers * case.n * sh.chunk_bytes
        configs = []
        if which in ("all", "kernels"):
            for stage, stages, cps, lag in [(32768, 6, 1, 3), (32768, 6, 1, 2), (32768, 6, 1, 4),
                                            (49152, 4, 1, 2), (49152, 4, 1, 1), (65536, 3, 1, 1),
                                            (40960, 5, 1, 2), (24576, 8, 1, 4), (16384, 12, 1, 6),
                                            (16384, 6, 2, 3), (32768, 3, 2, 1), (8192, 6, 4, 3)]:
                configs.append(dict(kernel=wk.KERNEL_TMA, stage_bytes=stage, stages=stages,
                                    ctas_per_sm=cps, store_lag=lag))
            for stage, cps in [(32768, 4), (65536, 2), (131072, 4)]:
                configs.append(dict(kernel=wk.KERNEL_SIMT, stage_bytes=stage, stages=6, ctas_per_sm=cps))
            for ef in (True,):
                configs.append(dict(kernel=wk.KERNEL_TMA, stage_bytes=32768, stages=6, ctas_per_sm=1,
                                    evict_first=ef))
        for cfg in configs:
            wk.set_tuning(wk.PATH_INTRA, **cfg)
            ms = timeit(lambda: wk.migrate(src, sbt, dst, dbt, stream=s), s)
            gbs = pb / ms / 1e6
            r = dict(case=name, **cfg, ms=round(ms, 3), gbs=round(gbs, 1), frac=round(2 * gbs / PEAK, 4))
            print(json.dumps(r), flush=True)
        wk.set_tuning(wk.PATH_INTRA, kernel=wk.KERNEL_TMA, stage_bytes=32768, stages=6, ctas_per_sm=1)
        if which in ("all", "stream") and name == "C2":
            cons = torch.cuda.Stream(dev)
            L = sh.n_layers

            def streamed(wait):
                for l in range(L):
                    wk.migrate(src, sbt, dst, dbt, layer_lo=l, layer_hi=l + 1, stream=s)
                if wait:
                    t = dst.layer_ticket()
                    for l in range(L):
                        wk.layer_wait(dst, l, t, stream=cons)
                    s.wait_stream(cons)
            for wait in (False, True):
                ms = timeit(lambda: streamed(wait), s, reps=5)
                print(json.dumps(dict(case=name, mode="streamed", wait=wait, ms=round(ms, 3),
                                      gbs=round(pb / ms / 1e6, 1))), flush=True)
            # one layer alone: launch + ramp + drain cost
            ms1 = timeit(lambda: wk.migrate(src, sbt, dst, dbt, layer_lo=5, layer_hi=6, stream=s), s, reps=20)
            print(json.dumps(dict(case=name, mode="one_layer", ms=round(ms1, 4),
                                  gbs=round(pb / L / ms1 / 1e6, 1))), flush=True)
            # CTA cap curve (for interference control)
            for cap in (8, 16, 24, 32, 48, 74, 148):
                wk.set_tuning(wk.PATH_INTRA, kernel=wk.KERNEL_TMA, max_ctas=cap)
                ms = timeit(lambda: wk.migrate(src, sbt, dst, dbt, stream=s), s, reps=3)
                print(json.dumps(dict(case=name, mode="cap", max_ctas=cap, gbs=round(pb / ms / 1e6, 1))),
                      flush=True)
            wk.set_tuning(wk.PATH_INTRA, kernel=wk.KERNEL_TMA, max_ctas=0)
        del src, dst
        torch.cuda.empty_cache()
    # copy-engine comparators
    n = 8 << 30
    a = torch.empty(n, dtype=torch.uint8, device=dev)
    b = torch.empty(n, dtype=torch.uint8, device=dev)
    ms = timeit(lambda: b.copy_(a), torch.cuda.current_stream(dev))
    print(json.dumps(dict(mode="torch_copy_8GiB", gbs_rw=round(2 * n / ms / 1e6, 1))), flush=True)
    ms = timeit(lambda: torch.cuda.current_stream(dev) and
                torch.cuda.cudart() and b.copy_(a, non_blocking=True), torch.cuda.current_stream(dev))


if __name__ == "__main__":
    main()
