#!/usr/bin/env python
"""bench.py — paged KV-migration throughput on B200 (BJ:metric "KV migration GB/s
(fraction of NVLink/HBM roofline) at 1/2/4/8 B200").

Step = one pass of the hot path over one batch: migrate a whole C2 workload (OPT-13B KV,
64 requests, ShareGPT-fit lengths 256-2048) from a prefill pool to a decode
pool through its block tables, all 40 layers, with per-layer completion flags (one
wind_kv_migrate call = one persistent kernel launch).
  N = 1 : both pools on cuda:0 (HBM-bound intra-device migration).
  N > 1 : ranks pair up 2k -> 2k+1; the source rank imports the decode rank's pool (CUDA
          IPC handles exchanged over a gloo process group) and pushes over NVLink peer
          stores.  An odd last rank runs the N = 1 step.  Weak scaling: every pair moves
          its own C2 workload.
`value` = payload bytes (K+V, all layers, whole blocks; table bytes excluded, reading R14)
of all ranks / max-over-ranks device time.  Extra scenarios (--scenarios, on by default at
N = 1) report the other §8(a) rows: layer-streamed hand-off, sequential tables,
compaction (C5), host swap (C1) — each with its own GB/s and roofline fraction.

--impl reference times the CPU oracle (oracle/, plain C, memcpy per chunk on all host
cores) on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "KV migration GB/s (fraction of NVLink/HBM roofline) at 1/2/4/8 B200"
LENGTH_MIX = {"C1": "512 tok each", "C2": "ShareGPT-fit 256-2048 tok", "C3": "2048 tok each",
              "C4": "LongBench-fit 16-4096 tok", "C5": "long-tail lognormal 16-8192 tok"}
GiB = 1 << 30


def load_peaks() -> dict:
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return {"hbm_gbs": float(d["hbm_gbs"]), "src": "measured", "sm_max_mhz": d.get("sm_max_mhz")}
    return {"hbm_gbs": 6650.0, "src": "fallback", "sm_max_mhz": 1965.0}


# ------------------------------------------------------------------------ clocks

class ClockSampler:
    """nvidia-smi sampling DURING the timed region (B200_PROFILING.md clocks line)."""

    Q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap,power.draw")

    def __init__(self, device: int):
        self.device = device
        self.proc = None
        self.lines: list[str] = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits", "-lms", "50",
                 "-i", str(self.device)], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self._t = threading.Thread(target=self._read, daemon=True)
            self._t.start()
            # nvidia-smi takes ~0.5-1 s to start: wait for its first sample, so the timed
            # region that follows is sampled from its start (bounded wait)
            t_end = time.time() + 5.0
            while not self.lines and time.time() < t_end and self.proc.poll() is None:
                time.sleep(0.01)
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append((time.time(), line.strip()))  # host arrival time (~ms)

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self, t0: float = 0.0, t1: float = float("inf")) -> dict:
        """Median SM clock and power, and every throttle reason seen, over the samples that
        arrived in host time [t0, t1] (default: all)."""
        sm, pw, mx, reasons = [], [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for t, ln in list(self.lines):
            if not t0 <= t <= t1:
                continue
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 6:
                continue
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
            except ValueError:
                continue
            for n, v in zip(names, f[2:6]):
                if v.lower().startswith("active"):
                    reasons.add(n)
            try:
                pw.append(float(f[6]))
            except (IndexError, ValueError):
                pass
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm),
                "power_w": round(float(np.median(pw)), 1) if pw else None}


# ----------------------------------------------------------------------- helpers

def payload_bytes(n_blocks: int, n_layers: int, chunk: int) -> int:
    """P5 closed form: 2 (K, V) x layers x blocks x C."""
    return 2 * n_layers * n_blocks * chunk


def make_pool(wk, shape, nb, device, seed, tag, loc="device"):
    import windgen.cuda as wg
    p = wk.Pool(shape.n_layers, shape.n_kv_heads, shape.head_dim, shape.block_size,
                shape.elem_bytes, nb, loc=loc, device=device)
    if loc == "device":
        wg.fill(p.base, p.nbytes, 0, seed, tag)
    return p


def time_device(fn, steps: int, warmup: int, stream, barrier=None, per_step=None):
    """W untimed warm-up steps, then EXACTLY `steps` steps between CUDA events on `stream`,
    barrier + synchronize on both sides.  Returns total ms.  With a list `per_step`, an
    event is also recorded between steps and the per-step ms are appended to it."""
    import torch
    for _ in range(warmup):
        fn()
    torch.cuda.synchronize()
    if barrier:
        barrier()
    ev = [torch.cuda.Event(enable_timing=True) for _ in range(steps + 1 if per_step is not None else 2)]
    ev[0].record(stream)
    for i in range(steps):
        fn()
        if per_step is not None:
            ev[i + 1].record(stream)
    ev[-1].record(stream)
    torch.cuda.synchronize()
    if barrier:
        barrier()
    if per_step is not None:
        per_step += [ev[i].elapsed_time(ev[i + 1]) for i in range(steps)]
    return ev[0].elapsed_time(ev[-1])


# ------------------------------------------------------------------ cpu baseline

def cpu_baseline(case, n_sample_blocks: int = 160, min_seconds: float = 10.0) -> dict:
    """The oracle as it stands (or_migrate_mt: T threads memcpy a static partition of the
    chunk list) on host DRAM pools, bounded sample of the same workload."""
    import oracle as O
    sh = case.shape
    n = min(n_sample_blocks, case.n)
    nb = math.ceil(1.1 * n)
    gs = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nb)
    src = np.ones(gs.pool_bytes, np.uint8)
    dst = np.zeros(gs.pool_bytes, np.uint8)
    sbt = np.random.default_rng(1).permutation(nb)[:n].astype(np.int32)
    dbt = np.random.default_rng(2).permutation(nb)[:n].astype(np.int32)
    T = O.hw_threads()
    O.migrate_mt(src, gs, sbt, dst, gs, dbt, 0, sh.n_layers, T)  # warm (page faults)
    reps, t0 = 0, time.perf_counter()
    while True:
        rc = O.migrate_mt(src, gs, sbt, dst, gs, dbt, 0, sh.n_layers, T)
        assert rc == O.OK
        reps += 1
        el = time.perf_counter() - t0
        if el >= min_seconds or reps >= 200:
            break
    byts = payload_bytes(n, sh.n_layers, sh.chunk_bytes) * reps
    return {"value": round(byts / el / 1e9, 3), "unit": "GB/s", "cores": T, "kind": "oracle",
            "sample": f"{n} of {case.n} C2 blocks ({payload_bytes(n, sh.n_layers, sh.chunk_bytes) / GiB:.2f} "
                      f"GiB payload) x {reps} reps, {el:.1f} s, or_migrate_mt with {T} threads"}


def parity_sample(wk, case, src, dst, lo, hi, n_check: int = 96) -> dict:
    """Sampled bit-exact check of the bench's own output (outside the timed region):
    the oracle gives each sampled destination chunk's origin (P2 closed form), windgen
    gives that origin's bytes."""
    import oracle as O
    import torch
    from windgen import content_bytes
    sh = case.shape
    gs = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, case.nb_src)
    gd = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, case.nb_dst)
    from_src, off = O.expected_origin(gs, case.src_bt, gd, case.dst_bt, lo, hi)
    rng = np.random.default_rng(7)
    touched = np.flatnonzero(from_src)
    idle = np.flatnonzero(from_src == 0)
    pick = np.concatenate([rng.choice(touched, min(n_check, touched.size), replace=False),
                           rng.choice(idle, min(n_check // 4, idle.size), replace=False)])
    C = sh.chunk_bytes
    t = dst.tensor()
    bad = 0
    for c in pick.tolist():
        got = t[c * C:(c + 1) * C].cpu().numpy()
        tag = case.src_tag if from_src[c] else case.dst_tag
        want = content_bytes(case.content_seed, tag, int(off[c]), C)
        bad += int(not np.array_equal(got, want))
    torch.cuda.synchronize()
    return {"chunks_checked": int(pick.size), "mismatches": bad, "ok": bad == 0}


# --------------------------------------------------------------------- scenarios

def run_scenarios(wk, device, peaks, steps=10, warmup=3) -> dict:
    """The other §8(a) rows on one GPU, each timed on its own stream with CUDA events."""
    import torch
    from windgen import (migration_case, SHAPES, live_mask_after_free, skewed_placement,
                         request_lengths, blocks_for_tokens)
    out = {}
    dev = torch.device("cuda", device)
    s = torch.cuda.Stream(device)
    hbm = peaks["hbm_gbs"]

    # (0) C1 intra-device (BJ:configs[0], S§8(d) C1 (i)): migrate pool A -> pool B, and
    #     compact pool A after a seeded half of its 8 requests is freed.  The working set
    #     (2 x 144 MiB) is ~2.3 x L2, so the L2 is flushed (a READ of 2 x l2CacheSize:
    #     clean lines, so no write-backs spill into the timed op) before every timed op,
    #     outside its events.
    out["c1_intra"] = run_c1_intra(wk, device, peaks, reps=20, warmup=warmup)

    # (1) C2 sequential tables (long runs: the coalescing / TMA best case)
    case = migration_case("C2", variant="sequential")
    sh = case.shape
    src = make_pool(wk, sh, case.nb_src, device, case.content_seed, case.src_tag)
    dst = make_pool(wk, sh, case.nb_dst, device, case.content_seed, case.dst_tag)
    sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
    pb = payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
    ms = time_device(lambda: wk.migrate(src, sbt, dst, dbt, stream=s), steps, warmup, s) / steps
    gbs = pb / ms / 1e6
    out["c2_sequential"] = {"gbs": round(gbs, 1), "hbm_frac": round(2 * gbs / hbm, 3), "ms": round(ms, 3)}
    del src, dst

    # (2) C2 shuffled, layer-streamed hand-off: 40 calls (lo = l, hi = l + 1), a consumer
    #     stream waits on each layer's flag (A5)
    case = migration_case("C2")
    src = make_pool(wk, sh, case.nb_src, device, case.content_seed, case.src_tag)
    dst = make_pool(wk, sh, case.nb_dst, device, case.content_seed, case.dst_tag)
    sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
    cons = torch.cuda.Stream(device)

    def streamed():
        for l in range(sh.n_layers):
            wk.migrate(src, sbt, dst, dbt, layer_lo=l, layer_hi=l + 1, stream=s)
        t = dst.layer_ticket()
        for l in range(sh.n_layers):
            wk.layer_wait(dst, l, t, stream=cons)
        s.wait_stream(cons)
    pb = payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
    ms = time_device(streamed, steps, warmup, s) / steps
    gbs = pb / ms / 1e6
    out["c2_layer_streamed"] = {"gbs": round(gbs, 1), "hbm_frac": round(2 * gbs / hbm, 3),
                                "ms": round(ms, 3), "launches_per_step": sh.n_layers}

    # copy-engine comparator on the same C2 gather (S§7 step 4): one cudaMemcpyAsync per
    # chunk (the classic per-block swap loop); host tables
    import victim
    planes = 2 * sh.n_layers

    def ce():
        victim.ce_gather("loop", src.base, case.nb_src * sh.chunk_bytes, dst.base,
                         case.nb_dst * sh.chunk_bytes, sh.chunk_bytes, case.src_bt, case.dst_bt,
                         planes, s.cuda_stream)
    ms = time_device(ce, 1, 2, s)
    gbs = pb / ms / 1e6
    out["c2_copy_engine_loop"] = {"gbs": round(gbs, 1), "hbm_frac": round(2 * gbs / hbm, 3),
                                  "ms": round(ms, 3), "copies": planes * case.n}
    del src, dst

    # (3) C5 compaction on GPU 0's share of the skewed placement (A7)
    pb, ms, moves, pool_gib = run_c5_compaction(wk, device, 0, 5 * steps, warmup)
    gbs = pb / ms / 1e6
    out["c5_compact"] = {"gbs": round(gbs, 1), "hbm_frac": round(2 * gbs / hbm, 3), "ms": round(ms, 3),
                         "moves": moves, "pool_gib": pool_gib}

    # (4) C1 host swap round trip over PCIe (A6): swap_out then swap_in at other slots
    case = migration_case("C1")
    sh1 = case.shape
    dpool = make_pool(wk, sh1, case.nb_src, device, case.content_seed, case.src_tag)
    dpool2 = make_pool(wk, sh1, case.nb_dst, device, case.content_seed, case.dst_tag)
    hpool = wk.Pool(sh1.n_layers, sh1.n_kv_heads, sh1.head_dim, sh1.block_size, sh1.elem_bytes,
                    case.n, loc="host")
    # default HOST path (SM / TMA kernel over mapped pinned memory, tables read when the op
    # runs) with a device host-side table, and the opt-in staged copy-engine path (kernel 4,
    # host-side table in pinned memory, read at enqueue)
    hbt_h = torch.arange(case.n, dtype=torch.int32).pin_memory()
    hbt = torch.arange(case.n, dtype=torch.int32, device=dev)
    sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
    pb = payload_bytes(case.n, sh1.n_layers, sh1.chunk_bytes)
    pcie = 63.0
    res = {}
    saved_h = wk.get_tuning(wk.PATH_HOST)
    for mech, ht, kern in (("sm_mapped", hbt, wk.KERNEL_AUTO), ("staged_ce", hbt_h, wk.KERNEL_STAGED)):
        wk.set_tuning(wk.PATH_HOST, **{**saved_h, "kernel": kern})
        ms_o = time_device(lambda: wk.swap_out(dpool, sbt, hpool, ht, stream=s), steps, warmup, s) / steps
        ms_i = time_device(lambda: wk.swap_in(hpool, ht, dpool2, dbt, stream=s), steps, warmup, s) / steps
        res[mech] = (pb / ms_o / 1e6, pb / ms_i / 1e6)
    wk.set_tuning(wk.PATH_HOST, **saved_h)
    (o, i), (o_st, i_st) = res["sm_mapped"], res["staged_ce"]
    out["c1_swap"] = {"out_gbs": round(o, 2), "in_gbs": round(i, 2),
                      "pcie_gen5_frac_out": round(o / pcie, 3), "pcie_gen5_frac_in": round(i / pcie, 3),
                      "mechanism": "default: TMA kernel stores to / loads from mapped pinned host memory",
                      "staged_ce_out_gbs": round(o_st, 2), "staged_ce_in_gbs": round(i_st, 2),
                      "staged_ce_mechanism": "opt-in kernel 4: TMA gather/scatter <-> device staging, "
                                             "copy engines over PCIe",
                      "payload_mib": round(pb / (1 << 20), 1), "pcie_peak_gbs": pcie}
    # copy-engine comparator (the practical PCIe ceiling)
    hbuf = torch.empty(pb, dtype=torch.uint8, pin_memory=True)
    dbuf = torch.empty(pb, dtype=torch.uint8, device=dev)
    ms_ce = time_device(lambda: hbuf.copy_(dbuf, non_blocking=True), steps, warmup,
                        torch.cuda.current_stream(device)) / steps
    out["c1_swap"]["copy_engine_d2h_gbs"] = round(pb / ms_ce / 1e6, 2)
    ms_ce = time_device(lambda: dbuf.copy_(hbuf, non_blocking=True), steps, warmup,
                        torch.cuda.current_stream(device)) / steps
    out["c1_swap"]["copy_engine_h2d_gbs"] = round(pb / ms_ce / 1e6, 2)
    del dpool, dpool2, hpool, hbuf, dbuf
    torch.cuda.empty_cache()

    # (5) interference with a co-running decode stream (C3): decode attention alone (the
    #     worst case: every byte of the step is KV), then a whole decode step (GEMMs too)
    out["c3_interference"] = run_interference(wk, device, peaks)
    torch.cuda.empty_cache()
    out["c3_interference_decode_step"] = run_interference(wk, device, peaks, victim_kind="decode_step")
    torch.cuda.empty_cache()

    # (6) stall-free rescheduling of P:120's request (NEXT-1)
    out["stall_free"] = run_stall_free(wk, device)
    torch.cuda.empty_cache()

    # (7) layer-streamed hand-off overlapped with a running prefill (NEXT-2)
    out["prefill_overlap_handoff"] = run_handoff(wk, device)
    torch.cuda.empty_cache()

    # (8) C4 memory pressure: evict by swap vs by migration, swap concurrent with hand-off
    out["c4_pressure"] = run_pressure(wk, device)
    torch.cuda.empty_cache()

    # (9) NEXT-4 policy: Eq. 2 fitted on the decode kernel, theta, trigger, victims
    out["policy_eq2"] = run_policy_profile(wk, device)
    torch.cuda.empty_cache()

    # (10) NEXT-3 backups (read-once fan-out) and TP reshard (head-range migrate)
    out["next3_backup_reshard"] = run_next3(wk, device, peaks)
    torch.cuda.empty_cache()
    return out


def run_c5_compaction(wk, device, gpu_index, steps, warmup, barrier=None):
    """A7 on GPU `gpu_index`'s share of C5's skewed placement over 8 GPUs: free a seeded
    half of its requests, plan_compact, compact.  Returns (payload bytes, ms per op, moves,
    pool GiB).  Repeating the op re-copies identical bytes (same traffic): that is timed."""
    import torch
    from windgen import (SHAPES, live_mask_after_free, skewed_placement, request_lengths,
                         blocks_for_tokens)
    dev = torch.device("cuda", device)
    s = torch.cuda.Stream(device)
    sh5 = SHAPES["C5"]
    lens = request_lengths("C5")
    place = skewed_placement(lens.size, 8, 4005)
    reqb = blocks_for_tokens(lens[place == gpu_index % 8], 16)
    nb = math.ceil(int(reqb.sum()) * 1.1)
    live, _ = live_mask_after_free(nb, reqb, 0.5, 4006 + gpu_index)
    csrc, cdst = wk.plan_compact(live)
    pool = make_pool(wk, sh5, nb, device, 3005, 1 + gpu_index)
    ts, td = torch.as_tensor(csrc, device=dev), torch.as_tensor(cdst, device=dev)
    pb = payload_bytes(len(csrc), sh5.n_layers, sh5.chunk_bytes)
    ms = time_device(lambda: wk.compact(pool, ts, td, stream=s), steps, warmup, s, barrier) / steps
    gib = round(pool.nbytes / GiB, 2)
    del pool
    return pb, ms, int(len(csrc)), gib


def run_c1_intra(wk, device, peaks, reps=20, warmup=3, replicas=8) -> dict:
    """C1 (BJ:configs[0], S§8(d)): the intra-device migrate pool A -> pool B (144 MiB) and the
    compaction of pool A after freeing half its requests, each measured two ways (the single
    op is the primary number, as in round 1):

    * single op: one op between two CUDA events with the L2 flushed (read of 2 x L2) before
      it.  This includes the fixed cost of ANY launch measured this way — an empty kernel
      between two events after the same flush measures `event_floor_us` (~5 us on B200,
      profiles/r02/launch_floor_probe.txt) — so a 12 us op can reach at most ~0.7 of HBM.
    * stream of cold ops: `replicas` independent pool pairs (R x 394 MB >> L2), ops issued
      back to back round-robin over them, one event pair around K ops: every op reads cold
      data (its pools were last touched R - 1 ops earlier), and the launch of op k + 1
      overlaps op k (programmatic dependent launch), as in a serving engine that issues
      migrations / compactions on a side stream.  Per-op time = window / K."""
    import torch
    from windgen import migration_case, live_mask_after_free, request_lengths, blocks_for_tokens
    dev = torch.device("cuda", device)
    s = torch.cuda.Stream(device)
    hbm = peaks["hbm_gbs"]
    case = migration_case("C1")
    sh = case.shape
    pairs = [(make_pool(wk, sh, case.nb_src, device, case.content_seed + 100 * r, case.src_tag),
              make_pool(wk, sh, case.nb_dst, device, case.content_seed + 100 * r, case.dst_tag))
             for r in range(replicas)]
    a, b = pairs[0]
    sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
    l2 = int(getattr(torch.cuda.get_device_properties(device), "L2_cache_size", 0) or (126 << 20))
    flush = torch.ones(2 * l2 // 4, dtype=torch.int32, device=dev)
    tiny = torch.zeros(1, device=dev)

    def timed(fn):
        for _ in range(warmup):
            fn()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
        torch.cuda.synchronize()
        with torch.cuda.stream(s):
            for e0, e1 in ev:
                flush.sum(dtype=torch.int64)  # evicts both pools' lines (untimed)
                e0.record(s)
                fn()
                e1.record(s)
        torch.cuda.synchronize()
        return float(np.median([e0.elapsed_time(e1) for e0, e1 in ev]))

    def stream_of_ops(op, k=8 * replicas):
        ms = time_device(lambda: [op(i) for i in range(k)], 3, 1, s) / 3
        return ms / k
    pb = payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
    floor_ms = timed(lambda: tiny.add_(0))
    ms = timed(lambda: wk.migrate(a, sbt, b, dbt, stream=s))
    ms_st = stream_of_ops(lambda i: wk.migrate(pairs[i % replicas][0], sbt, pairs[i % replicas][1], dbt, stream=s))
    res = {"migrate_gbs": round(pb / ms / 1e6, 1), "migrate_hbm_frac": round(2 * pb / ms / 1e6 / hbm, 3),
           "migrate_ms": round(ms, 4),
           "migrate_stream_gbs": round(pb / ms_st / 1e6, 1),
           "migrate_stream_hbm_frac": round(2 * pb / ms_st / 1e6 / hbm, 3),
           "migrate_stream_ms_per_op": round(ms_st, 4), "payload_mib": round(pb / (1 << 20), 1),
           "event_floor_us": round(floor_ms * 1e3, 2),
           "l2_flush_read_bytes_before_each_single_op": int(flush.numel() * 4),
           "stream_replicas": replicas,
           "stream_working_set_mib": round(replicas * (a.nbytes + b.nbytes) / (1 << 20))}
    reqb = blocks_for_tokens(request_lengths("C1"), sh.block_size)
    live, _ = live_mask_after_free(case.nb_src, reqb, 0.5, 4001)
    csrc, cdst = wk.plan_compact(live)
    ts, td = torch.as_tensor(csrc, device=dev), torch.as_tensor(cdst, device=dev)
    pc = payload_bytes(len(csrc), sh.n_layers, sh.chunk_bytes)
    ms = timed(lambda: wk.compact(a, ts, td, stream=s))
    ms_st = stream_of_ops(lambda i: wk.compact(pairs[i % replicas][0], ts, td, stream=s))
    res.update({"compact_moves": int(len(csrc)), "compact_gbs": round(pc / ms / 1e6, 1),
                "compact_hbm_frac": round(2 * pc / ms / 1e6 / hbm, 3), "compact_ms": round(ms, 4),
                "compact_single_op_ceiling_frac": round(2 * pc / hbm / 1e3 / (2 * pc / hbm / 1e3 + floor_ms * 1e3), 3),
                "compact_stream_gbs": round(pc / ms_st / 1e6, 1),
                "compact_stream_hbm_frac": round(2 * pc / ms_st / 1e6 / hbm, 3),
                "compact_stream_ms_per_op": round(ms_st, 4),
                "note": "*_hbm_frac / *_ms: one op between CUDA events after an L2 flush; it "
                        "includes the event_floor_us that an empty launch costs in the same "
                        "measurement, so compact_single_op_ceiling_frac = ideal / (ideal + floor) "
                        "bounds it; *_stream_*: ops back to back round-robin over "
                        "stream_replicas pool pairs (data >> L2), window / ops"})
    del a, b, pairs, flush
    return res


def run_next3(wk, device, peaks, steps=10, warmup=3) -> dict:
    """NEXT-3 (P:233 backups; P:128 / Table 3 mismatched TP placements), C2 geometry at half
    size (1452 blocks, 17.7 GiB):
    * backup fan-out: the same blocks into TWO destination pools.  read_once = one launch
      whose items share one source table (the TMA kernel stages each unit once and stores it
      twice: 3 x payload of DRAM traffic); per_item = one launch, separate table objects
      (each item re-reads the source: 4 x payload); two_launches = two migrates.
    * TP-2 -> TP-1 reshard: two half-head (20 of 40 heads) source pools pushed into one
      full pool at head offsets 0 and 20 (wind_kv_migrate_heads, 80 KiB spans)."""
    import torch
    from windgen import migration_case, KVShape, SHAPES
    sh = SHAPES["C2"]
    dev = torch.device("cuda", device)
    s = torch.cuda.Stream(device)
    hbm = peaks["hbm_gbs"]
    case = migration_case("C2", scale=0.5)
    src = make_pool(wk, sh, case.nb_src, device, case.content_seed, case.src_tag)
    a = make_pool(wk, sh, case.nb_dst, device, case.content_seed, case.dst_tag)
    b = make_pool(wk, sh, case.nb_dst, device, case.content_seed, case.dst_tag + 1)
    sbt = torch.as_tensor(case.src_bt, device=dev)
    sbt2 = sbt.clone()
    dbt = torch.as_tensor(case.dst_bt, device=dev)
    pb = payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
    out = {"blocks": case.n, "payload_gib_per_destination": round(pb / GiB, 2)}
    runs = {"read_once": lambda: wk.migrate_batch(src, [(a, sbt, dbt), (b, sbt, dbt)], 0, sh.n_layers, stream=s),
            "per_item": lambda: wk.migrate_batch(src, [(a, sbt, dbt), (b, sbt2, dbt)], 0, sh.n_layers, stream=s),
            "two_launches": lambda: (wk.migrate(src, sbt, a, dbt, stream=s), wk.migrate(src, sbt, b, dbt, stream=s))}
    for name, fn in runs.items():
        ms = time_device(fn, steps, warmup, s) / steps
        dram = (3 if name == "read_once" else 4) * pb
        out[f"fanout2_{name}"] = {"ms": round(ms, 3), "delivered_gbs": round(2 * pb / ms / 1e6, 1),
                                  "dram_gbs": round(dram / ms / 1e6, 1),
                                  "hbm_frac": round(dram / ms / 1e6 / hbm, 3)}
    del src, a, b
    torch.cuda.empty_cache()
    half = KVShape("OPT-13B TP-2 shard", sh.n_layers, sh.n_kv_heads // 2, sh.head_dim, sh.elem_bytes)
    shards = [make_pool(wk, half, case.nb_src, device, case.content_seed, 40 + r) for r in range(2)]
    full = make_pool(wk, sh, case.nb_dst, device, case.content_seed, 50)

    def reshard():
        for r, sp in enumerate(shards):
            wk.migrate_heads(sp, sbt, full, dbt, 0, r * half.n_kv_heads, half.n_kv_heads, stream=s)
    ms = time_device(reshard, steps, warmup, s) / steps
    out["tp2_to_tp1_reshard"] = {"ms": round(ms, 3), "gbs": round(pb / ms / 1e6, 1),
                                 "hbm_frac": round(2 * pb / ms / 1e6 / hbm, 3),
                                 "span_kib": half.n_kv_heads * sh.block_size * sh.head_dim * sh.elem_bytes // 1024}
    del shards, full
    return out


def run_handoff(wk, device, cap_ctas: int = 16, n_tokens: int = 2048, reps: int = 5) -> dict:
    """NEXT-2 ("overlapping KV transfers with prefill computation"): an
    OPT-13B prefill of one 2048-token request runs layer by layer (the 24*N*H^2 GEMM FLOPs
    of Table 1 per layer, as bf16 cuBLAS matmuls on the prefill stream); as soon
    as layer l is computed, an event releases migrate(layer l) on the migration stream, and
    the decode side waits on layer_done[l].  Reported: prefill slowdown caused by the
    overlapped transfer, and the hand-off latency (prefill end -> last layer landed)
    overlapped vs. transferring everything after the prefill.  Migration capped at
    `cap_ctas` CTAs (~NVLink rate)."""
    import torch
    from windgen import SHAPES
    sh = SHAPES["C2"]
    H = sh.n_kv_heads * sh.head_dim  # hidden size 5120
    L, bs = sh.n_layers, sh.block_size
    dev = torch.device("cuda", device)
    nblk = -(-n_tokens // bs)
    src = make_pool(wk, sh, nblk + 8, device, 1, 1)
    dst = make_pool(wk, sh, nblk + 8, device, 1, 2)
    sbt = torch.arange(nblk, dtype=torch.int32, device=dev)
    dbt = torch.arange(8, 8 + nblk, dtype=torch.int32, device=dev)
    x = torch.randn(n_tokens, H, device=dev, dtype=torch.bfloat16)
    w_qkv = torch.randn(H, 3 * H, device=dev, dtype=torch.bfloat16) * 0.01
    w_o = torch.randn(H, H, device=dev, dtype=torch.bfloat16) * 0.01
    w_1 = torch.randn(H, 4 * H, device=dev, dtype=torch.bfloat16) * 0.01
    w_2 = torch.randn(4 * H, H, device=dev, dtype=torch.bfloat16) * 0.01
    pre, mig, cons = torch.cuda.Stream(device), torch.cuda.Stream(device), torch.cuda.Stream(device)
    saved = wk.get_tuning(wk.PATH_INTRA)
    wk.set_tuning(wk.PATH_INTRA, **{**saved, "max_ctas": cap_ctas})

    def layer_compute():
        with torch.cuda.stream(pre):
            qkv = x @ w_qkv
            a = qkv[:, :H] @ w_o
            h = a @ w_1
            return h @ w_2

    def run(mode: str):
        """mode: 'alone' (prefill only), 'overlap' (per-layer migration), 'serial'."""
        evs = [torch.cuda.Event() for _ in range(L)]
        t_start, t_pre_end, t_landed = (torch.cuda.Event(enable_timing=True) for _ in range(3))
        torch.cuda.synchronize()
        t_start.record(pre)
        for l in range(L):
            layer_compute()
            evs[l].record(pre)
            if mode == "overlap":
                mig.wait_event(evs[l])
                wk.migrate(src, sbt, dst, dbt, layer_lo=l, layer_hi=l + 1, stream=mig)
        t_pre_end.record(pre)
        if mode == "serial":
            mig.wait_event(evs[L - 1])
            wk.migrate(src, sbt, dst, dbt, stream=mig)
        if mode != "alone":
            t = dst.layer_ticket()
            for l in range(L):
                wk.layer_wait(dst, l, t, stream=cons)
            t_landed.record(cons)
        torch.cuda.synchronize()
        pre_ms = t_start.elapsed_time(t_pre_end)
        land = t_pre_end.elapsed_time(t_landed) if mode != "alone" else 0.0
        return pre_ms, land

    for _ in range(2):
        run("overlap")
    res = {}
    for mode in ("alone", "overlap", "serial"):
        vals = [run(mode) for _ in range(reps)]
        res[mode] = (float(np.median([v[0] for v in vals])), float(np.median([v[1] for v in vals])))
    wk.set_tuning(wk.PATH_INTRA, **saved)
    flops = 24 * n_tokens * H * H * L
    return {"request_tokens": n_tokens, "cap_ctas": cap_ctas,
            "prefill_ms_alone": round(res["alone"][0], 3),
            "prefill_tflops_alone": round(flops / res["alone"][0] / 1e9, 1),
            "prefill_ms_with_overlapped_transfer": round(res["overlap"][0], 3),
            "prefill_slowdown": round(res["overlap"][0] / res["alone"][0] - 1, 4),
            "handoff_latency_ms_overlapped": round(res["overlap"][1], 3),
            "handoff_latency_ms_serial": round(res["serial"][1], 3),
            "kv_bytes": payload_bytes(nblk, L, sh.chunk_bytes)}


def run_pressure(wk, device, reps: int = 3) -> dict:
    """C4 (Llama-2-70B GQA bf16, 32 LongBench-fit requests per pair) under memory pressure
    (S§8(d)): the decode pool holds resident requests and must take an incoming batch; it
    can only hold 0.8 x (resident + incoming), so victims (longest first) must
    leave.  DistServe swaps them to host; WindServe reschedules them to the
    prefill instance.  Measured: time to evict the victims by swap-out (PCIe)
    vs by migration (HBM here; NVLink-rate cap 16 CTAs and uncapped), and the incoming
    hand-off running concurrently with the swap-out (separate links, separate streams)."""
    import torch
    from windgen import SHAPES, lengths_longbench, blocks_for_tokens
    sh = SHAPES["C4"]
    dev = torch.device("cuda", device)
    res_b = blocks_for_tokens(lengths_longbench(32, 1004), 16)
    inc_b = blocks_for_tokens(lengths_longbench(32, 2004), 16)
    n_res, n_inc = int(res_b.sum()), int(inc_b.sum())
    cap = int(0.8 * (n_res + n_inc))
    need = n_res + n_inc - cap
    order = np.argsort(-res_b, kind="stable")            # longest first, lowest id on ties
    take = np.cumsum(res_b[order]) < need
    take[np.argmin(take)] = True                           # the request that crosses `need`
    victims = order[take]
    starts = np.concatenate([[0], np.cumsum(res_b)])
    vic_slots = np.concatenate([np.arange(starts[r], starts[r + 1]) for r in victims]).astype(np.int32)
    nv = vic_slots.size
    dpool = make_pool(wk, sh, cap, device, 3004, 1)         # resident in slots [0, n_res)
    host = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nv, loc="host")
    other = make_pool(wk, sh, nv + 8, device, 3004, 2)      # the prefill instance's pool
    src_inc = make_pool(wk, sh, n_inc + 8, device, 3004, 3)
    s_swap, s_mig = torch.cuda.Stream(device), torch.cuda.Stream(device)
    vt = torch.as_tensor(vic_slots, device=dev)
    ht = torch.arange(nv, dtype=torch.int32, device=dev)
    ht_h = torch.arange(nv, dtype=torch.int32).pin_memory()  # host slots (default SM path)
    free_now = cap - n_res
    inc_src = torch.arange(n_inc, dtype=torch.int32, device=dev)
    inc_dst = torch.as_tensor(np.concatenate([np.arange(n_res, cap), vic_slots])[:n_inc].astype(np.int32),
                              device=dev)
    vb = payload_bytes(nv, sh.n_layers, sh.chunk_bytes)
    ib = payload_bytes(n_inc, sh.n_layers, sh.chunk_bytes)
    t_swap = time_device(lambda: wk.swap_out(dpool, vt, host, ht_h, stream=s_swap), reps, 2, s_swap) / reps
    saved = wk.get_tuning(wk.PATH_INTRA)
    out = {"victims": int(victims.size), "victim_gib": round(vb / GiB, 2), "incoming_gib": round(ib / GiB, 2),
           "evict_by_swap_ms": round(t_swap, 2), "swap_gbs": round(vb / t_swap / 1e6, 1)}
    for capc in (16, 0):
        wk.set_tuning(wk.PATH_INTRA, **{**saved, "max_ctas": capc})
        t_m = time_device(lambda: wk.migrate(dpool, vt, other, ht, stream=s_mig), reps, 2, s_mig) / reps
        out[f"evict_by_migration_ms_cap{capc or 'none'}"] = round(t_m, 3)
    wk.set_tuning(wk.PATH_INTRA, **saved)
    # concurrent: swap the victims out while the incoming batch lands in the free slots; the
    # part that needs victim slots waits for the swap-out (an event after swap_out)
    k_free = min(free_now, n_inc)

    def both():
        ev = torch.cuda.Event()
        wk.swap_out(dpool, vt, host, ht_h, stream=s_swap)
        ev.record(s_swap)
        wk.migrate(src_inc, inc_src[:k_free], dpool, inc_dst[:k_free], stream=s_mig)
        if n_inc > k_free:
            s_mig.wait_event(ev)
            wk.migrate(src_inc, inc_src[k_free:], dpool, inc_dst[k_free:], stream=s_mig)
        s_mig.wait_stream(s_swap)
    t_both = time_device(both, reps, 1, s_mig) / reps
    out["swap_out_plus_incoming_ms"] = round(t_both, 2)
    out["paper_claim"] = ("rescheduling (migration) instead of swapping frees the decode pool "
                          f"{t_swap / out['evict_by_migration_ms_cap16']:.0f}x faster at an NVLink-rate cap")
    # full-duplex PCIe: swap the victims out to a second host pool while the first host
    # pool's copy (the earlier victims) swaps back in, on two streams (DistServe-style swap
    # traffic both ways at once, P:130 / P:341); aggregate = both directions' payload
    host2 = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nv, loc="host")
    back_t = torch.as_tensor(np.arange(nv, dtype=np.int32), device=dev)

    def exchange():
        s_swap.wait_stream(s_mig)
        wk.swap_out(dpool, vt, host2, ht_h, stream=s_swap)
        wk.swap_in(host, ht_h, other, back_t, stream=s_mig)
        s_mig.wait_stream(s_swap)
    t_x = time_device(exchange, reps, 1, s_mig) / reps
    out["swap_exchange"] = {"ms": round(t_x, 2), "aggregate_gbs": round(2 * vb / t_x / 1e6, 1),
                            "note": "swap-out and swap-in of 12.7 GiB each at the same time (default SM paths)"}
    # the same eviction and exchange through the opt-in staged copy-engine path (kernel 4:
    # host tables read on the CPU at enqueue; the pinned host-slot table ht_h)
    saved_h = wk.get_tuning(wk.PATH_HOST)
    wk.set_tuning(wk.PATH_HOST, **{**saved_h, "kernel": wk.KERNEL_STAGED})
    try:
        t_sw_st = time_device(lambda: wk.swap_out(dpool, vt, host, ht_h, stream=s_swap), reps, 1, s_swap) / reps
        t_x_st = time_device(exchange, reps, 1, s_mig) / reps
    finally:
        wk.set_tuning(wk.PATH_HOST, **saved_h)
    out["staged_opt_in"] = {"swap_gbs": round(vb / t_sw_st / 1e6, 1),
                            "swap_exchange_aggregate_gbs": round(2 * vb / t_x_st / 1e6, 1)}
    host2.destroy()
    del dpool, host, other, src_inc
    return out


def run_policy_profile(wk, device, bw_gbs: float = 550.0) -> dict:
    """NEXT-4: the Profiler's Eq. 2 (T_decode = a_d * sum(L) + c_d) fitted on the
    decode-attention kernel over OPT-13B KV (40 layers) at sum(L) = 8K..128K tokens, then the
    stall-free threshold theta it implies (R6) and the trigger / victim choice for a
    decode pool at 97 % occupancy (R7, R8)."""
    import torch
    import victim
    from paper_conf_isca_fenghzly025_b200 import policy
    from windgen import SHAPES, lengths_sharegpt, blocks_for_tokens
    sh = SHAPES["C2"]
    dev = torch.device("cuda", device)
    bs = sh.block_size
    max_tok = 2048
    s = torch.cuda.Stream(device)
    xs, ys = [], []
    nb = 64 * max_tok // bs
    pool = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, 2, nb, device=device)
    pool.tensor().view(torch.float16).normal_()
    plane = nb * sh.chunk_bytes
    for B in (4, 8, 16, 32, 64):
        bt = torch.randperm(nb)[:B * max_tok // bs].to(torch.int32).view(B, -1).to(dev)
        ctx = torch.full((B,), max_tok, dtype=torch.int32, device=dev)
        q = torch.randn(B, sh.n_kv_heads, 128, device=dev, dtype=torch.float16)
        scratch = torch.empty(victim.scratch_floats(B, sh.n_kv_heads, max_tok // bs, 64), device=dev)
        out = torch.empty(B, sh.n_kv_heads, 128, device=dev)

        def step():
            for l in range(sh.n_layers):
                kp = pool.base + 2 * l * plane
                victim.decode_attention(q, kp, kp + plane, bt, ctx, sh.n_kv_heads, bs, scratch, out,
                                        blocks_per_split=64, stream=s.cuda_stream)
        ms = time_device(step, 10, 3, s) / 10
        xs.append(B * max_tok)
        ys.append(ms)
    a, c, r2 = policy.fit_decode_profile(xs, ys)
    # a decode pool at 97 % occupancy holding 64 ShareGPT-length requests
    reqb = blocks_for_tokens(lengths_sharegpt(64, 77), bs)
    n_pool = int(math.ceil(reqb.sum() / 0.97))
    free = n_pool - int(reqb.sum())
    trig = policy.should_reschedule(free, n_pool, new_blocks_per_step=len(reqb))
    need = int(0.05 * n_pool) - free + len(reqb)
    vic = policy.pick_victims(reqb, need)
    sum_L = float(reqb.sum() * bs)
    theta = policy.theta_from_profile(a, c, sum_L, bw_gbs, sh.n_layers, sh.chunk_bytes)
    del pool
    return {"eq2_points_sumL_ms": [[int(x), round(y, 3)] for x, y in zip(xs, ys)],
            "a_d_us_per_token": round(a * 1e3, 5), "c_d_ms": round(c, 4), "r2": round(r2, 5),
            "pool_blocks": n_pool, "free_blocks": free, "trigger": bool(trig),
            "victims": vic, "victim_blocks": int(reqb[vic].sum()) if vic else 0,
            "theta_blocks_at_bw_gbs": {"bw_gbs": bw_gbs, "theta": theta},
            "note": "decode attention only (Table 1's 4*SUM(L)*H KV read, P:162); GEMMs omitted"}


def run_stall_free(wk, device, cap_ctas: int = 16) -> dict:
    """NEXT-1: one OPT-13B request of 2048 tokens (1.5625 GiB of KV) keeps
    decoding while it migrates; it is blocked only for the final stage.  The migration is
    capped at `cap_ctas` CTAs (~700 GB/s, an NVLink-rate push) and compared with a
    stop-the-world migration of the same request at the same rate."""
    import torch
    from paper_conf_isca_fenghzly025_b200 import stall_free
    from windgen import SHAPES
    import windgen.cuda as wg
    sh = SHAPES["C2"]
    bs, T0, nb, capb = sh.block_size, 2048, 600, 300
    dev = torch.device("cuda", device)
    rng = np.random.default_rng(0)
    ss = rng.permutation(nb)[:capb].astype(np.int32)
    ds = rng.permutation(nb)[:capb].astype(np.int32)
    src = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb, device=device)
    dst = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb, device=device)
    wg.fill(src.base, src.nbytes, 0, 1, 1)
    saved = wk.get_tuning(wk.PATH_INTRA)
    wk.set_tuning(wk.PATH_INTRA, **{**saved, "max_ctas": cap_ctas})
    mig, dec = torch.cuda.Stream(device), torch.cuda.Stream(device)
    st, dt = torch.as_tensor(ss, device=dev), torch.as_tensor(ds, device=dev)
    step = stall_free.append_token_kernel_factory(src, ss, dec)
    step(T0)
    torch.cuda.synchronize()
    # decode-step time of the synthetic append and the stop-the-world migration time
    t0 = time.perf_counter()
    for t in range(T0, T0 + 20):
        step(t)
        dec.synchronize()
    step_ms = (time.perf_counter() - t0) / 20 * 1e3
    n0 = T0 // bs
    stw = time_device(lambda: wk.migrate(src, st, dst, dt, n=n0, stream=mig), 3, 2, mig) / 3
    bw = n0 * 2 * sh.n_layers * sh.chunk_bytes / stw / 1e6
    theta = stall_free.default_theta(max(step_ms, 0.05), bw, sh.n_layers, sh.chunk_bytes)
    res = stall_free.migrate_stall_free(src, st, dst, dt, T0, theta, step, mig, dec)
    wk.set_tuning(wk.PATH_INTRA, **saved)
    # the same request with its stages issued as full-rate bursts of 8 blocks (100 MiB) per
    # decode step (chunk_blocks; the interference rows show why: burst vs trickle)
    resb = stall_free.migrate_stall_free(src, st, dst, dt, T0 + 64, theta, step, mig, dec, chunk_blocks=8)
    del src, dst
    return {"request": "OPT-13B, 2048 tokens at start (P:120)", "cap_ctas": cap_ctas,
            "migration_gbs": round(bw, 1), "stop_the_world_ms": round(stw, 3),
            "theta_blocks": theta, "stages": len(res.stages), "tokens_decoded_while_migrating":
            int(sum(res.appends)), "pause_ms": round(res.pause_ms, 3),
            "blocked_time_reduction": round(1 - res.pause_ms / stw, 4),
            "blocks_sent": res.blocks_sent,
            "bursts_of_8_blocks_per_decode_step": {
                "stages": len(resb.stages), "tokens_decoded_while_migrating": int(sum(resb.appends)),
                "pause_ms": round(resb.pause_ms, 3), "blocks_sent": resb.blocks_sent}}


def make_victim(wk, device, peaks, victim_kind="attention", n_steps=50):
    """The co-running decode work of the interference measurements (S§8(d)), as one CUDA
    graph per step on a HIGH-priority stream (plus a LOW-priority stream for the migration):
    "attention" = paged decode attention over 16 x 2048 resident tokens of OPT-66B KV (the
    Fig. 8 decode set; 72 GiB read per step), "decode_step" = a whole OPT-66B decode
    step on one TP-2 rank (QKV, attention over 36 heads, output projection, MLP; fp16 cuBLAS
    GEMMs on one layer's 1.02 GB weight shard re-read every layer).  Returns a namespace
    with the graph, the streams, run(n) (per-step events), step_on(stream) (to capture it
    elsewhere), t_alone (median step ms) and info (description, HBM fraction)."""
    import types
    import torch
    import victim
    from windgen import migration_case, SHAPES, KVShape
    sh = SHAPES["C3"]
    dev = torch.device("cuda", device)
    B, ctx_len, bs = 16, 2048, sh.block_size
    nbv = B * ctx_len // bs
    full_step = victim_kind == "decode_step"
    vsh = KVShape("OPT-66B TP-2 shard", sh.n_layers, sh.n_kv_heads // 2, sh.head_dim, sh.elem_bytes) \
        if full_step else sh
    vpool = wk.Pool(vsh.n_layers, vsh.n_kv_heads, vsh.head_dim, bs, vsh.elem_bytes, nbv, device=device)
    vt = vpool.tensor().view(torch.float16)
    g = torch.Generator(device=dev).manual_seed(0)
    step_elems = 1 << 28
    for o in range(0, vt.numel(), step_elems):
        n = min(step_elems, vt.numel() - o)
        vt[o:o + n].normal_(generator=g)
    perm = torch.randperm(nbv, generator=torch.Generator().manual_seed(1)).to(torch.int32)
    bt = perm.view(B, ctx_len // bs).to(dev)
    ctx = torch.full((B,), ctx_len, dtype=torch.int32, device=dev)
    hv = vsh.n_kv_heads
    q = torch.randn(B, hv, sh.head_dim, device=dev, dtype=torch.float16)
    bps = 64  # sweep r01: 0.978 of HBM on this shape
    scratch = torch.empty(victim.scratch_floats(B, hv, ctx_len // bs, bps), device=dev)
    out = torch.empty(B, hv, sh.head_dim, device=dev)
    plane = nbv * vsh.chunk_bytes
    hi_s = torch.cuda.Stream(device, priority=-1)
    lo_s = torch.cuda.Stream(device, priority=0)
    if full_step:  # one TP-2 layer's weight shard, fp16, re-read by every layer
        Hd, Hs = 9216, hv * sh.head_dim  # hidden size of OPT-66B, this rank's attention width
        gw = torch.Generator(device=dev).manual_seed(2)
        w_qkv = torch.randn(Hd, 3 * Hs, device=dev, dtype=torch.float16, generator=gw) * 0.01
        w_o = torch.randn(Hs, Hd, device=dev, dtype=torch.float16, generator=gw) * 0.01
        w_1 = torch.randn(Hd, 2 * Hd, device=dev, dtype=torch.float16, generator=gw) * 0.01
        w_2 = torch.randn(2 * Hd, Hd, device=dev, dtype=torch.float16, generator=gw) * 0.01
        h0 = torch.randn(B, Hd, device=dev, dtype=torch.float16, generator=gw)
        w_bytes = sum(w.numel() * 2 for w in (w_qkv, w_o, w_1, w_2))

    def victim_step_on(st):
        if not full_step:
            for l in range(sh.n_layers):
                kp = vpool.base + (2 * l) * plane
                victim.decode_attention(q, kp, kp + plane, bt, ctx, hv, bs, scratch, out,
                                        blocks_per_split=bps, stream=st.cuda_stream)
            return
        with torch.cuda.stream(st):
            h = h0
            for l in range(sh.n_layers):
                qkv = h @ w_qkv
                ql = qkv[:, :Hs].contiguous().view(B, hv, sh.head_dim)
                kp = vpool.base + (2 * l) * plane
                victim.decode_attention(ql, kp, kp + plane, bt, ctx, hv, bs, scratch, out,
                                        blocks_per_split=bps, stream=st.cuda_stream)
                h1 = h + out.view(B, Hs).half() @ w_o
                h = torch.tanh(h1 + torch.nn.functional.gelu(h1 @ w_1) @ w_2)

    def victim_step():
        victim_step_on(hi_s)

    for _ in range(5):
        victim_step()
    torch.cuda.synchronize()
    # a decode step is one CUDA-graph replay (as serving engines run it): its 128 launches
    # cannot be delayed by host-side contention with the thread that enqueues migrations
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph, stream=hi_s):
        victim_step()
    torch.cuda.synchronize()

    def victim_run(n, g=None, st=None):
        g, st = g or graph, st or hi_s
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(n + 1)]
        with torch.cuda.stream(st):
            ev[0].record(st)
            for i in range(n):
                g.replay()
                ev[i + 1].record(st)
        return ev
    ev = victim_run(n_steps)
    torch.cuda.synchronize()
    alone = [ev[i].elapsed_time(ev[i + 1]) for i in range(n_steps)]
    t_alone = float(np.median(alone))
    kv_read = B * ctx_len * sh.n_layers * 2 * hv * sh.head_dim * sh.elem_bytes
    step_bytes = kv_read + (w_bytes * sh.n_layers if full_step else 0)
    info = {"victim_ms_alone": round(t_alone, 3),
           "victim_hbm_frac": round(step_bytes / t_alone / 1e6 / peaks["hbm_gbs"], 3),
           "victim": ("OPT-66B decode step on one TP-2 rank: QKV, paged attention (36 heads, "
                      "16 x 2048 tok), output projection, MLP; 64 layers; weights "
                      f"{w_bytes * sh.n_layers / 1e9:.1f} GB + KV {kv_read / 1e9:.1f} GB per step"
                      if full_step else "paged decode attention, 16 x 2048 tok, 64 layers, 72 heads (C3)")}

    return types.SimpleNamespace(graph=graph, hi_s=hi_s, lo_s=lo_s, run=victim_run, step_on=victim_step_on,
                                 t_alone=t_alone, info=info, pool=vpool, sh=sh, dev=dev)


def run_interference(wk, device, peaks, n_victim_steps=50, configs=None, victim_kind="attention") -> dict:
    """S§8(d) interference, C3 (OPT-66B KV, 64 layers x 72 heads x d 128, fp16): the victim
    is paged decode attention over 16 x 2048 resident tokens (the Fig. 8 decode set,
    P:251) = 72 GiB of KV read per step (64 layer launches) on a HIGH-priority stream; the
    migration moves 4 x 2048-token long-context requests (P:227, 18 GiB) on a LOW-priority
    side stream, looped to cover every victim step.  On one GPU the migration is
    intra-device (reads AND writes this HBM); a CTA cap emulates the source-side HBM load
    of an NVLink push (8 CTAs ~ 365 GB/s payload = 730 GB/s of DRAM traffic, about what a
    770 GB/s peer push reads on its source GPU).

    victim_kind="decode_step": a victim closer to a whole decode step of OPT-66B on one
    TP-2 rank (Table 3 placements are TP-2): per layer the QKV projection, paged
    attention over this rank's 36 heads of the 16 x 2048-token set, the output projection
    and the MLP — fp16 GEMMs (cuBLAS, harness only) against one layer's weight shard
    (1.02 GB, re-read every layer: it cannot stay in the 126 MB L2) — so a step streams
    65 GB of weights plus 36 GiB of KV."""
    import torch
    from windgen import migration_case
    V = make_victim(wk, device, peaks, victim_kind, n_victim_steps)
    sh, dev = V.sh, V.dev
    graph, hi_s, lo_s, victim_step_on, victim_run, t_alone = V.graph, V.hi_s, V.lo_s, V.step_on, V.run, V.t_alone
    full_step = victim_kind == "decode_step"
    res = dict(V.info)

    case = migration_case("C3")
    src = make_pool(wk, sh, case.nb_src, device, case.content_seed, case.src_tag)
    dst = make_pool(wk, sh, case.nb_dst, device, case.content_seed, case.dst_tag)
    d_tabs = (torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev))
    h_tabs = (torch.as_tensor(case.src_bt).pin_memory(), torch.as_tensor(case.dst_bt).pin_memory())
    pb = payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
    saved = wk.get_tuning(wk.PATH_INTRA)
    saved_host = wk.get_tuning(wk.PATH_HOST)
    n_sw = min(64, case.n)  # host-swap loads: 64 of the case's blocks (2.25 GiB), looped
    host = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, n_sw, loc="host")
    sw_dev = torch.as_tensor(case.src_bt[:n_sw], device=dev)
    sw_host = {"dev": torch.arange(n_sw, dtype=torch.int32, device=dev),
               "pinned": torch.arange(n_sw, dtype=torch.int32).pin_memory()}
    # push-source proxy: a 1-block destination pool (36 MiB, L2-resident); its table maps
    # every source block to slot 0 — duplicate destinations, outside the table contract on
    # purpose (the bytes are never read; release builds do not check table content)
    sink = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, 1, device=device)
    zeros_t = torch.zeros(case.n, dtype=torch.int32, device=dev)
    if configs is None and full_step:  # the whole-decode-step victim: the informative rows
        configs = ([("control_no_migration", {**saved, "null_feeder": True}),
                    ("cap2", {**saved, "max_ctas": 2})] +
                   [(f"rate{r}GBs", {**saved, "max_ctas": 0, "rate_mbps": r * 1000}) for r in (50, 150)] +
                   [("copy_engines_rate50GBs", {**saved, "kernel": wk.KERNEL_COPY_ENGINE, "rate_mbps": 50000}),
                    ("swap_out_sm_default", {"op": "swap_out", **saved_host, "kernel": wk.KERNEL_TMA}),
                    ("push_source_proxy_rate700GBs", {**saved, "op": "push_source_proxy", "max_ctas": 0,
                                                      "rate_mbps": 700000})])
    configs = configs or (
        [("control_no_migration", {**saved, "null_feeder": True})] +
        [(f"cap{c or 'none'}", {**saved, "max_ctas": c}) for c in (2, 4, 8, 16, 0)] +
        [(f"rate{r}GBs", {**saved, "max_ctas": 0, "rate_mbps": r * 1000}) for r in (50, 100, 150, 300)] +
        [(f"rate{r}GBs_32ctas", {**saved, "max_ctas": 32, "rate_mbps": r * 1000}) for r in (100,)] +
        # L2 evict-first on the migration's loads and stores: the streamed KV should not push
        # the victim's small hot data (block tables, queries, partial outputs) out of L2
        [(f"rate{r}GBs_evict_first", {**saved, "max_ctas": 0, "rate_mbps": r * 1000, "evict_first": 1})
         for r in (50, 150)] +
        [("cap2_evict_first", {**saved, "max_ctas": 2, "evict_first": 1})] +
        [(f"copy_engines_rate{r}GBs", {**saved, "kernel": wk.KERNEL_COPY_ENGINE, "rate_mbps": r * 1000})
         for r in (50, 100, 150, 300)] +
        # SM partition (green contexts, wind_kv_partition_sms): migration confined to 8 SMs,
        # the victim on the other 140 — no migration CTA ever shares an SM with the victim
        [("partition8_tma", {**saved, "partition": 8, "max_ctas": 0}),
         ("partition8_tma_rate50GBs", {**saved, "partition": 8, "max_ctas": 0, "rate_mbps": 50000}),
         ("partition8_tma_rate150GBs", {**saved, "partition": 8, "max_ctas": 0, "rate_mbps": 150000})] +
        # host swaps (A6) next to the decode victim: the SM kernel on mapped pinned memory (HBM
        # one way only: swap out reads, swap in writes) at the library's per-direction CTA
        # defaults, the swap-out at the former 8-CTA default (PCIe write backpressure), and the
        # staged copy-engine path (gather / scatter through the staging buffer + DMA)
        [("swap_out_sm_default", {"op": "swap_out", **saved_host, "kernel": wk.KERNEL_TMA}),
         ("swap_out_sm_8ctas", {"op": "swap_out", **saved_host, "kernel": wk.KERNEL_TMA, "max_ctas": 8}),
         ("swap_in_sm_default", {"op": "swap_in", **saved_host, "kernel": wk.KERNEL_TMA}),
         ("swap_out_staged", {"op": "swap_out", **saved_host, "kernel": wk.KERNEL_STAGED}),
         ("swap_in_staged", {"op": "swap_in", **saved_host, "kernel": wk.KERNEL_STAGED})] +
        # SOURCE side of an NVLink push, emulated on one GPU: the migration reads its source
        # blocks from this HBM at the link's rate, and its stores all land in ONE destination
        # block (36 MiB over all layers: they stay in L2), so this HBM sees the push's reads
        # and almost none of its writes — what a prefill GPU pushing to a peer sees.  A proxy
        # (no NVLink traffic, the source-side HBM load only), labelled as such.
        [(f"push_source_proxy_rate{r}GBs", {**saved, "op": "push_source_proxy", "max_ctas": 0,
                                            "rate_mbps": r * 1000}) for r in (350, 700)] +
        [("push_source_proxy_uncapped", {**saved, "op": "push_source_proxy", "max_ctas": 0})])
    rounds, n_round = 3, max(10, n_victim_steps // 2)
    part = {}  # SM partition (green contexts): victim graph on the compute SMs
    clk = ClockSampler(device).__enter__()  # SM clock / power per phase (power-cap effects)
    time.sleep(1.0)  # nvidia-smi start-up

    def partitioned(min_sms):
        if min_sms not in part:
            P = wk.Partition(device, min_sms)
            g = torch.cuda.CUDAGraph()
            for _ in range(2):
                with torch.cuda.stream(P.compute):
                    victim_step_on(P.compute)
            torch.cuda.synchronize()
            with torch.cuda.graph(g, stream=P.compute):
                victim_step_on(P.compute)
            torch.cuda.synchronize()
            part[min_sms] = (P, g)
        return part[min_sms]
    for name, cfg in configs:
        cfg = dict(cfg)
        null = cfg.pop("null_feeder", False)  # control: the feeder thread runs, moves nothing
        min_sms = cfg.pop("partition", 0)
        op_kind = cfg.pop("op", "migrate")
        mig_s, vic_g, vic_s = lo_s, graph, hi_s
        if min_sms:
            P, vic_g = partitioned(min_sms)
            mig_s, vic_s = P.migration, P.compute
        if op_kind == "migrate":
            wk.set_tuning(wk.PATH_INTRA, **cfg)
            ce = cfg.get("kernel") == wk.KERNEL_COPY_ENGINE
            sbt, dbt = (h_tabs[0].data_ptr(), h_tabs[1].data_ptr()) if ce else d_tabs
            op_bytes = pb

            def one_op():
                wk.migrate(src, sbt, dst, dbt, n=case.n, stream=mig_s)
        elif op_kind == "push_source_proxy":
            wk.set_tuning(wk.PATH_INTRA, **cfg)
            op_bytes = pb

            def one_op():  # every source block -> destination block 0 (stays in L2)
                wk.migrate(src, d_tabs[0], sink, zeros_t, n=case.n, stream=mig_s)
        else:
            wk.set_tuning(wk.PATH_HOST, **cfg)
            ht = sw_host["pinned" if cfg.get("kernel") == wk.KERNEL_STAGED else "dev"]
            op_bytes = payload_bytes(n_sw, sh.n_layers, sh.chunk_bytes)
            if op_kind == "swap_out":
                def one_op():
                    wk.swap_out(src, sw_dev, host, ht, stream=mig_s)
            else:
                def one_op():
                    wk.swap_in(host, ht, src, sw_dev, stream=mig_s)
        t_mig = time_device(one_op, 2, 3, mig_s) / 2
        full_alone = []
        alone_all, with_all, covered = [], [], True
        win_alone, win_with = [], []
        co_bytes, co_secs = 0, 0.0
        # `rounds` interleaved pairs (victim alone, then victim + migration): the alone
        # reference is always adjacent in time (removes clock / power drift).  A feeder
        # thread keeps exactly one migration op in flight on the low-priority stream for the
        # whole victim run (the victim's launches are never queued behind migration work on
        # the host; ctypes releases the GIL inside the library calls).
        for _ in range(rounds):
            torch.cuda.synchronize()
            if min_sms:  # the whole-GPU reference too: the partition itself costs the victim SMs
                ev = victim_run(n_round)
                torch.cuda.synchronize()
                full_alone += [ev[i].elapsed_time(ev[i + 1]) for i in range(n_round)]
            ta0 = time.time()
            ev = victim_run(n_round, vic_g, vic_s)
            torch.cuda.synchronize()
            win_alone.append((ta0, time.time()))
            alone = [ev[i].elapsed_time(ev[i + 1]) for i in range(n_round)]
            stop, started, n_ops = threading.Event(), threading.Event(), [0]
            done_t: list = []  # host time of each op completion (migration rate while co-running)

            def feeder():
                while not stop.is_set():
                    if null:
                        started.set()
                        time.sleep(0.001)
                        continue
                    one_op()
                    started.set()
                    mig_s.synchronize()
                    done_t.append(time.time())
                    n_ops[0] += 1
            th = threading.Thread(target=feeder, daemon=True)
            th.start()
            started.wait()
            tw0 = time.time()
            ev = victim_run(n_round, vic_g, vic_s)
            torch.cuda.synchronize()
            tw1 = time.time()
            win_with.append((tw0, tw1))
            stop.set()
            th.join()
            ts = [t for t in done_t if tw0 <= t <= tw1]
            if len(ts) >= 2:
                co_bytes += op_bytes * (len(ts) - 1)
                co_secs += ts[-1] - ts[0]
            covered &= th is not None and n_ops[0] >= 1
            with_all += [ev[i].elapsed_time(ev[i + 1]) for i in range(n_round)]
            alone_all += alone
        t_ref, t_with = float(np.median(alone_all)), float(np.median(with_all))
        # HBM bytes per payload byte: intra-device read + write; SM swap one way; the staged
        # swap adds its gather / scatter through the staging buffer (3 ways)
        hbm_ways = 2 if op_kind == "migrate" else (3 if cfg.get("kernel") == wk.KERNEL_STAGED else 1)  # proxy: reads
        res[name] = {
            "migration_gbs_alone": round(op_bytes / t_mig / 1e6, 1),
            "migration_hbm_share": round(hbm_ways * op_bytes / t_mig / 1e6 / peaks["hbm_gbs"], 4),
            "victim_ms_alone_adjacent": round(t_ref, 3),
            "victim_ms_with_migration": round(t_with, 3),
            "slowdown": round(t_with / t_ref - 1.0, 4),
            # the migration's own rate WHILE the victim runs (ops completed inside the victim
            # window; None when fewer than 2 completed there, e.g. slow rate-limited ops)
            "migration_gbs_during": round(co_bytes / co_secs / 1e9, 1) if co_secs > 0 else None,
            "migration_covered_all_victim_steps": bool(covered)}

        def phase(wins):
            sm, pw, rs = [], [], set()
            for a_, b_ in wins:
                c_ = clk.summary(a_, b_)
                if c_["sm_mhz"] is not None:
                    sm.append(c_["sm_mhz"])
                if c_["power_w"] is not None:
                    pw.append(c_["power_w"])
                rs |= set(c_["reasons"])
            return {"sm_mhz": float(np.median(sm)) if sm else None,
                    "power_w": round(float(np.median(pw)), 1) if pw else None, "reasons": sorted(rs)}
        res[name]["clocks_alone"] = phase(win_alone)
        res[name]["clocks_with_migration"] = phase(win_with)
        if min_sms:
            t_full = float(np.median(full_alone))
            res[name].update({"partition_sms_migration": P.sms_migration, "partition_sms_compute": P.sms_compute,
                              "victim_ms_alone_whole_gpu": round(t_full, 3),
                              "slowdown_vs_whole_gpu": round(t_with / t_full - 1.0, 4)})
    # Burst instead of trickle: the same AVERAGE migration rate delivered as one full-rate op
    # per decode step, released by an event at the step's start (the op overlaps the first
    # part of the step), against the rate-limited trickle rows above.  A trickle holds HBM
    # (and SMs) for the whole step; a burst finishes early and leaves the rest of the step
    # alone, so the victim's added time per migrated byte can differ.
    wk.set_tuning(wk.PATH_INTRA, **saved)
    blk_bytes = payload_bytes(1, sh.n_layers, sh.chunk_bytes)
    for avg, proxy in ((50, False), (150, False), (300, False), (700, True)):
        nb_step = max(1, min(case.n, round(avg * 1e9 * t_alone * 1e-3 / blk_bytes)))
        sb_ = d_tabs[0][:nb_step]
        db_, dpool_ = (zeros_t[:nb_step], sink) if proxy else (d_tabs[1][:nb_step], dst)
        t_b = time_device(lambda: wk.migrate(src, sb_, dpool_, db_, n=nb_step, stream=lo_s), 3, 2, lo_s) / 3

        def burst_run(n):
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(n + 1)]
            ev[0].record(hi_s)
            for i in range(n):
                go = torch.cuda.Event()
                go.record(hi_s)
                lo_s.wait_event(go)
                wk.migrate(src, sb_, dpool_, db_, n=nb_step, stream=lo_s)
                with torch.cuda.stream(hi_s):
                    graph.replay()
                ev[i + 1].record(hi_s)
            return ev
        alone_b, with_b = [], []
        for _ in range(rounds):
            torch.cuda.synchronize()
            ev = victim_run(n_round)
            torch.cuda.synchronize()
            alone_b += [ev[i].elapsed_time(ev[i + 1]) for i in range(n_round)]
            ev = burst_run(n_round)
            torch.cuda.synchronize()
            with_b += [ev[i].elapsed_time(ev[i + 1]) for i in range(n_round)]
        tr, tw = float(np.median(alone_b)), float(np.median(with_b))
        res[f"burst_{'push_source_proxy_' if proxy else ''}avg{avg}GBs"] = {
            "blocks_per_step": int(nb_step), "mb_per_step": round(nb_step * blk_bytes / 1e6, 1),
            "avg_gbs": round(nb_step * blk_bytes / tr / 1e6, 1), "burst_ms_alone": round(t_b, 3),
            "victim_ms_alone_adjacent": round(tr, 3), "victim_ms_with_migration": round(tw, 3),
            "slowdown": round(tw / tr - 1.0, 4),
            "note": "one full-rate op per decode step, released at the step's start"}
    # The library's step-aligned op (wind_kv_migrate_stepped): slices released by the
    # victim's own step signal (wind_kv_step_signal before each step's graph replay), the
    # whole migration enqueued up front on the low-priority stream.
    counter = torch.zeros(1, dtype=torch.int32, device=dev)
    issued = [0]
    for avg, proxy in ((50, False), (150, False), (250, True), (400, True)):
        bps = int(avg * 1e9 * t_alone * 1e-3)
        dpool_, db_ = (sink, zeros_t) if proxy else (dst, d_tabs[1])

        def stepped_run(n):
            base, k = issued[0], 0
            while k < n:
                n0 = wk.launch_count()
                wk.migrate_stepped(src, d_tabs[0], dpool_, db_, counter, first_step=base + k + 1,
                                   bytes_per_step=bps, n=case.n, stream=lo_s)
                k += wk.launch_count() - n0
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(n + 1)]
            ev[0].record(hi_s)
            for i in range(n):
                wk.step_signal(counter, stream=hi_s)
                with torch.cuda.stream(hi_s):
                    graph.replay()
                ev[i + 1].record(hi_s)
            for _ in range(k - n):  # release the slices enqueued past the last step
                wk.step_signal(counter, stream=hi_s)
            issued[0] = base + k
            return ev
        alone_s, with_s = [], []
        for _ in range(rounds):
            torch.cuda.synchronize()
            ev = victim_run(n_round)
            torch.cuda.synchronize()
            alone_s += [ev[i].elapsed_time(ev[i + 1]) for i in range(n_round)]
            ev = stepped_run(n_round)
            torch.cuda.synchronize()
            with_s += [ev[i].elapsed_time(ev[i + 1]) for i in range(n_round)]
        tr, tw = float(np.median(alone_s)), float(np.median(with_s))
        res[f"stepped_{'push_source_proxy_' if proxy else ''}avg{avg}GBs"] = {
            "bytes_per_step": bps, "avg_gbs": round(bps / tr / 1e6, 1),
            "victim_ms_alone_adjacent": round(tr, 3), "victim_ms_with_migration": round(tw, 3),
            "slowdown": round(tw / tr - 1.0, 4),
            "note": "wind_kv_migrate_stepped: slices released by the victim's wind_kv_step_signal"}
    clk.__exit__()
    wk.set_tuning(wk.PATH_INTRA, **saved)
    wk.set_tuning(wk.PATH_HOST, **saved_host)
    torch.cuda.synchronize()
    for P, _ in part.values():
        P.destroy()
    host.destroy()
    del V, src, dst, sink
    return res


def run_all_to_all(wk, rank, world, device, peaks, steps=5, warmup=3, scale=1.0) -> dict:
    """A8 at N > 1: C5 (Llama-3-8B GQA fp8, 1024 long-tail requests) placed with skewed
    weights over the ranks; every rank derives the same plan (uniform hash shuffle =
    bandwidth headline; greedy rebalance = realistic), imports every peer's pool and pushes
    its outgoing blocks to all peers in one wind_kv_migrate_batch launch."""
    import torch
    import torch.distributed as dist
    from paper_conf_isca_fenghzly025_b200 import parallel, rebalance
    from windgen import (SHAPES, request_lengths, skewed_placement, blocks_for_tokens,
                         hash_shuffle_dest)
    sh = SHAPES["C5"]
    lens = request_lengths("C5", scale=scale)
    gpu = skewed_placement(lens.size, world, 4005)
    blocks = blocks_for_tokens(lens, 16).astype(np.int32)
    loads = np.bincount(gpu, weights=blocks, minlength=world).astype(np.int64)
    nb = int(loads.max() + math.ceil(1.5 * blocks.sum() / world))
    rng = [np.random.default_rng(5000 + g) for g in range(world)]
    perms = [r.permutation(nb) for r in rng]
    pos = [0] * world
    tables = []
    for r in range(lens.size):
        g = int(gpu[r])
        tables.append(perms[g][pos[g]:pos[g] + blocks[r]].astype(np.int32))
        pos[g] += int(blocks[r])
    free = []
    for g in range(world):
        m = np.ones(nb, bool)
        m[perms[g][:pos[g]]] = False
        free.append(m)
    dev = torch.device("cuda", device)
    pool = make_pool(wk, sh, nb, device, 3005, 10 + rank)
    handles = parallel.exchange_handles(pool.export())
    peers = {g: wk.Pool.import_(h, device) for g, h in enumerate(handles) if g != rank}
    s = torch.cuda.Stream(device)
    keep = []

    def to_dev(a):
        t = torch.as_tensor(a, device=dev)
        keep.append(t)
        return t
    out = {}
    for kind in ("shuffle", "rebalance"):
        if kind == "shuffle":
            plan = rebalance.plan_exchange(world, gpu, tables, free,
                                           hash_shuffle_dest(lens.size, world, 4005))
        else:
            plan = rebalance.plan_rebalance_exchange(world, gpu, tables, free)
        items = plan.items_for(rank)
        batch = [(peers[d], to_dev(sb), to_dev(db)) for d, sb, db in items]
        sent = sum(int(sb.size) for _, sb, _ in items)

        def step():
            for k in range(0, len(batch), wk.MAX_BATCH):
                wk.migrate_batch(pool, batch[k:k + wk.MAX_BATCH], 0, sh.n_layers, stream=s)
        if not batch:
            step = lambda: None  # noqa: E731
        ms = time_device(step, steps, warmup, s, barrier=dist.barrier) / steps
        ms_max, = parallel.max_over_ranks([ms])
        tot = plan.blocks_moved * 2 * sh.n_layers * sh.chunk_bytes
        per_gpu_egress = sent * 2 * sh.n_layers * sh.chunk_bytes / ms / 1e6
        out[kind] = {"aggregate_gbs": round(tot / ms_max / 1e6, 1), "ms": round(ms_max, 3),
                     "blocks_moved": int(plan.blocks_moved),
                     "rank0_egress_gbs": round(per_gpu_egress, 1) if rank == 0 else None,
                     "nvlink_frac_per_gpu": round(tot / world / ms_max / 1e6 / 770.0, 4),
                     "nvlink_frac_per_gpu_of_nominal_900": round(tot / world / ms_max / 1e6 / 900.0, 4)}
    for p in peers.values():
        p.destroy()
    return out


def run_peer_interference(wk, rank, world, device, peaks, rounds=3, n_steps=20) -> dict:
    """Interference on the REAL multi-GPU configuration (S§8(d); "decoding continues
    during migration"): every rank runs the whole-decode-step victim (make_victim
    "decode_step") while the prefill rank of each pair pushes C3 long-context KV into
    its partner's imported pool over NVLink — trickled at 150 GB/s (the burst pacer),
    uncapped, or as wind_kv_migrate_stepped slices released by the SOURCE rank's own decode
    steps (avg 150 / 400 GB/s).  Reported per side: the source (push) rank's victim reads
    only (its HBM serves the push's loads), the destination rank's victim sees the push's
    writes.  Each configuration is measured against an adjacent victim-alone run; slowdowns
    are the max over pairs.  With every rank on one GPU (WIND_BENCH_ONE_DEVICE) the code path
    runs but the numbers are not NVLink numbers."""
    import threading
    import torch
    import torch.distributed as dist
    from paper_conf_isca_fenghzly025_b200 import parallel
    from windgen import migration_case
    role, partner = parallel.pair_role(rank, world)
    V = make_victim(wk, device, peaks, "decode_step", n_steps)
    dev = torch.device("cuda", device)
    case = migration_case("C3")
    sh = case.shape
    src = dst = None
    if role == "push":
        src = make_pool(wk, sh, case.nb_src, device, case.content_seed, case.src_tag)
    if role == "decode":
        dst = make_pool(wk, sh, case.nb_dst, device, case.content_seed, case.dst_tag)
    handles = parallel.exchange_handles(dst.export() if role == "decode" else None)
    if role == "push":
        dst = wk.Pool.import_(handles[partner], device)
    sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
    pb = payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
    counter = torch.zeros(1, dtype=torch.int32, device=dev)
    issued = [0]

    path = wk.route(src, dst)[1] if role == "push" else wk.PATH_PEER  # PEER across GPUs
    saved = wk.get_tuning(path)

    def victim_with(kind, arg):
        """Runs n_steps of the victim on every rank; the push rank migrates alongside.
        Returns this rank's per-step ms."""
        stop, th = threading.Event(), None
        if role == "push" and kind in ("trickle", "uncapped"):
            wk.set_tuning(path, **{**saved, "rate_mbps": arg if kind == "trickle" else 0, "max_ctas": 0})

            def feeder():
                while not stop.is_set():
                    wk.migrate(src, sbt, dst, dbt, n=case.n, stream=V.lo_s)
                    V.lo_s.synchronize()
            th = threading.Thread(target=feeder, daemon=True)
            th.start()
            time.sleep(0.01)
        extra = 0
        if role == "push" and kind == "stepped":
            bps, k, base = int(arg * 1e6 * V.t_alone * 1e-3), 0, issued[0]
            while k < n_steps:
                n0 = wk.launch_count()
                wk.migrate_stepped(src, sbt, dst, dbt, counter, first_step=base + k + 1, bytes_per_step=bps,
                                   n=case.n, stream=V.lo_s)
                k += wk.launch_count() - n0
            extra = k - n_steps
            issued[0] = base + k
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(n_steps + 1)]
        ev[0].record(V.hi_s)
        for i in range(n_steps):
            if role == "push" and kind == "stepped":
                wk.step_signal(counter, stream=V.hi_s)
            with torch.cuda.stream(V.hi_s):
                V.graph.replay()
            ev[i + 1].record(V.hi_s)
        for _ in range(extra):
            wk.step_signal(counter, stream=V.hi_s)
        V.hi_s.synchronize()
        stop.set()
        if th is not None:
            th.join()
        torch.cuda.synchronize()
        wk.set_tuning(path, **saved)
        return [ev[i].elapsed_time(ev[i + 1]) for i in range(n_steps)]

    out = {"victim": V.info["victim"], "victim_ms_alone": V.info["victim_ms_alone"], "pairs": world // 2}
    for name, kind, arg in (("trickle150GBs", "trickle", 150000), ("uncapped", "uncapped", 0),
                            ("stepped_avg150GBs", "stepped", 150000), ("stepped_avg400GBs", "stepped", 400000)):
        alone, withm = [], []
        for _ in range(rounds):
            dist.barrier()
            alone += victim_with("alone", 0)
            dist.barrier()
            withm += victim_with(kind, arg)
        slow = float(np.median(withm)) / float(np.median(alone)) - 1.0
        # per side: max over the ranks of that role
        sides = [None] * world
        dist.all_gather_object(sides, (role, slow))
        src_s = [x for r, x in sides if r == "push"]
        dst_s = [x for r, x in sides if r == "decode"]
        out[name] = {"source_slowdown": round(max(src_s), 4) if src_s else None,
                     "destination_slowdown": round(max(dst_s), 4) if dst_s else None}
    out["payload_gib_per_op"] = round(pb / GiB, 2)
    if role == "push":
        dst.destroy()
    dist.barrier()
    del V, src, dst
    return out


# -------------------------------------------------------------------------- main# -------------------------------------------------------------------------- main

def run_gpu(args) -> None:
    import torch
    import torch.distributed as dist
    import paper_conf_isca_fenghzly025_b200 as wk
    from windgen import migration_case

    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    if os.environ.get("WIND_BENCH_ONE_DEVICE"):  # test hook: every rank on cuda:0 (CUDA IPC
        local = 0                                 # between processes on one GPU)
    if world != args.gpus:
        raise SystemExit(f"--gpus {args.gpus} but WORLD_SIZE={world}")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        import datetime
        # bounded: a rank that fails in a scenario must not hang the others forever
        dist.init_process_group("gloo", rank=rank, world_size=world,
                                timeout=datetime.timedelta(seconds=600))
    barrier = (lambda: dist.barrier()) if world > 1 else None
    peaks = load_peaks()

    from paper_conf_isca_fenghzly025_b200 import parallel
    case = migration_case(args.config, variant=args.variant, seed_offset=args.seed)
    sh = case.shape
    role, partner = parallel.pair_role(rank, world)
    src = dst = None
    if role in ("solo", "push"):
        src = make_pool(wk, sh, case.nb_src, local, case.content_seed, case.src_tag)
    if role in ("solo", "decode"):
        dst = make_pool(wk, sh, case.nb_dst, local, case.content_seed, case.dst_tag)
    if world > 1:
        # pair setup (CUDA IPC export / import): every rank reports whether it succeeded, so
        # a failure prints one explanatory line instead of a traceback and a hung barrier
        err = None
        try:
            # both pools of a pair are exported: the push rank imports the decode pool (push:
            # the prefill GPU's SMs store over NVLink), the decode rank imports the prefill
            # pool (pull: the decode GPU's SMs load over NVLink) — the autotune below times both
            handles = parallel.exchange_handles(dst.export() if role == "decode" else
                                                (src.export() if role == "push" else None))
            if role == "push":
                dst = wk.Pool.import_(handles[partner], local)
            elif role == "decode":
                src = wk.Pool.import_(handles[partner], local)
        except Exception as e:  # noqa: BLE001 — reported below, then the run ends
            err = f"rank {rank}: {type(e).__name__}: {e}"[:300]
        errs: list = [None] * world
        dist.all_gather_object(errs, err)
        errs = [x for x in errs if x]
        if errs:
            if rank == 0:
                print(json.dumps({"metric": METRIC, "value": None, "unit": "GB/s", "n_gpus": world,
                                  "error": "peer pool setup failed: " + " | ".join(errs)}), flush=True)
            dist.barrier()
            dist.destroy_process_group()
            raise SystemExit(1)
    stream = torch.cuda.Stream(local)
    sbt = torch.as_tensor(case.src_bt, device=dev)
    dbt = torch.as_tensor(case.dst_bt, device=dev)
    lo, hi = 0, sh.n_layers
    pb = payload_bytes(case.n, hi - lo, sh.chunk_bytes)

    # who executes a pair's op: "push" = the prefill rank (src local, dst imported), "pull" =
    # the decode rank (src imported, dst local); a solo rank always runs its own op
    mode = {"v": "push"}

    def executes() -> bool:
        return role == "solo" or (role == "push") == (mode["v"] == "push")

    def step():
        if executes():
            wk.migrate(src, sbt, dst, dbt, layer_lo=lo, layer_hi=hi, stream=stream)

    # N > 1: the peer-path kernel is chosen on the real link before the timed steps (round 1
    # never had two GPUs in one call, so the default was never measured over NVLink 5):
    # every candidate runs the same op for 3 steps (max over ranks), the fastest becomes the
    # PEER tuning for the headline.  Reported as `peer_autotune` in the line.
    peer_tune = None
    if world > 1:
        simt96 = dict(kernel=wk.KERNEL_SIMT, ctas_per_sm=1, stage_bytes=32768, stages=6, max_ctas=96)
        simt4 = dict(kernel=wk.KERNEL_SIMT, ctas_per_sm=4, stage_bytes=32768, stages=6)
        tma148 = dict(kernel=wk.KERNEL_TMA, ctas_per_sm=1, stage_bytes=49152, stages=4, store_lag=2)
        cands = [("push_simt_96ctas", "push", simt96), ("push_simt_4x148", "push", simt4),
                 ("push_tma_148", "push", tma148), ("push_tma_64", "push", {**tma148, "max_ctas": 64}),
                 ("push_tma_32", "push", {**tma148, "max_ctas": 32}),
                 ("pull_simt_4x148", "pull", simt4), ("pull_tma_148", "pull", tma148),
                 ("pull_tma_64", "pull", {**tma148, "max_ctas": 64})]
        default_peer = wk.get_tuning(wk.PATH_PEER)
        try:
            rates = {}
            for name, m, cfg in cands:
                mode["v"] = m
                wk.set_tuning(wk.PATH_PEER, **cfg)
                ms_alt, = parallel.max_over_ranks([time_device(step, 3, 3, stream, barrier) / 3])
                rates[name] = round(pb / ms_alt / 1e6, 1)
            best = max(rates, key=rates.get)
            _, mode["v"], cfg = next(c for c in cands if c[0] == best)
            wk.set_tuning(wk.PATH_PEER, **cfg)
            peer_tune = {"chosen": best, "gbs_per_pair": rates}
        except Exception as e:  # noqa: BLE001 — reported; the library default (push) stays
            mode["v"] = "push"
            wk.set_tuning(wk.PATH_PEER, **default_peer)
            peer_tune = {"error": f"{type(e).__name__}: {e}"[:300]}
            print(f"[bench rank {rank}] peer autotune failed: {peer_tune['error']}", file=sys.stderr, flush=True)
    torch.cuda.synchronize()
    launches0 = wk.launch_count()
    step_ms: list = []
    with ClockSampler(local) as clk:
        t_timed0 = time.time()
        ms_total = time_device(step, args.steps, args.warmup, stream, barrier, per_step=step_ms)
        t_timed1 = time.time()
        time.sleep(0.06)  # the sample covering the region's last 50 ms
    # the samples that arrived during the timed region (all samples if that window is too
    # short to hold three of them)
    clk_timed = clk.summary(t_timed0, t_timed1 + 0.06)
    if clk_timed["samples"] < 3:
        clk_timed = clk.summary()
    clk_timed["window_s"] = round(t_timed1 - t_timed0, 3)
    launches = wk.launch_count() - launches0 - (args.warmup if executes() else 0)
    if world > 1:  # every rank's library launches in the timed region (pull: the decode ranks')
        t_l = torch.tensor([float(launches)], dtype=torch.float64)
        dist.all_reduce(t_l)
        launches = int(t_l.item())
    ms_step_local = ms_total / args.steps
    # e2e: tables from pinned host memory H2D, the migrate, the layer flags read back D2H
    h_sbt = torch.as_tensor(case.src_bt).pin_memory()
    h_dbt = torch.as_tensor(case.dst_bt).pin_memory()
    d_sbt, d_dbt = torch.empty_like(sbt), torch.empty_like(dbt)
    flags_host = torch.empty(sh.n_layers, dtype=torch.int32).pin_memory()

    def e2e_step():
        if not executes():
            return
        with torch.cuda.stream(stream):
            d_sbt.copy_(h_sbt, non_blocking=True)
            d_dbt.copy_(h_dbt, non_blocking=True)
        wk.migrate(src, d_sbt, dst, d_dbt, layer_lo=lo, layer_hi=hi, stream=stream)
        dst.read_flags(flags_host, stream=stream)  # the step's result: layer_done[] D2H
        stream.synchronize()

    e2e_steps = max(3, args.steps // 2)
    ms_e2e_local = time_device(e2e_step, e2e_steps, args.warmup, stream, barrier) / e2e_steps

    ms_step, ms_e2e = parallel.max_over_ranks([ms_step_local, ms_e2e_local])
    n_movers = parallel.movers(world)
    total_bytes = pb * n_movers
    a2a = None
    compaction = None
    peer_interf = None
    scen_error = None
    if world > 1 and args.scenarios:
        # The multi-GPU scenarios never ran on more than one GPU in round 1 (one GPU per
        # gpurun call): a failure there is reported in the line, never loses the headline.
        try:
            torch.cuda.synchronize()
            del src, dst
            torch.cuda.empty_cache()
            a2a = run_all_to_all(wk, rank, world, local, peaks, scale=args.a2a_scale)
            # intra-device work at N GPUs (A7): every rank compacts its own share of C5 at
            # the same time (GPU g holds placement share g mod 8); aggregate = sum / max time
            pbc, msc, _, _ = run_c5_compaction(wk, local, rank, 10, 3, barrier=dist.barrier)
            tot_b = torch.tensor([float(pbc)], dtype=torch.float64)
            dist.all_reduce(tot_b)
            ms_c, = parallel.max_over_ranks([msc])
            compaction = {"aggregate_gbs": round(float(tot_b.item()) / ms_c / 1e6, 1), "ms_max": round(ms_c, 3),
                          "hbm_frac_per_gpu": round(2 * float(tot_b.item()) / world / ms_c / 1e6 / peaks["hbm_gbs"], 3)}
            torch.cuda.empty_cache()
            # the co-running decode step on the source and destination GPUs of NVLink pushes
            if args.peer_interference:
                peer_interf = run_peer_interference(wk, rank, world, local, peaks)
        except Exception as e:  # noqa: BLE001 — reported, not swallowed
            scen_error = f"{type(e).__name__}: {e}"[:400]
            print(f"[bench rank {rank}] multi-GPU scenario failed: {scen_error}", file=sys.stderr, flush=True)
    value = total_bytes / ms_step / 1e6  # GB/s
    e2e_value = total_bytes / ms_e2e / 1e6

    extra = {}
    if rank == 0:
        kernel_gbs = pb / ms_step / 1e6  # one mover's op (max over ranks: the executing rank)
        if role == "solo":
            roof = {"bound": "hbm", "achieved": round(2 * kernel_gbs, 1), "peak": peaks["hbm_gbs"],
                    "unit": "GB/s", "frac": round(2 * kernel_gbs / peaks["hbm_gbs"], 4),
                    "traffic": traffic_from_profiles(args.config), "peak_src": peaks["src"],
                    "per_launch_bytes": 2 * pb,
                    "note": "algorithmic DRAM bytes = 2 x payload (read + write) per launch; "
                            "1 launch (wind_kv tma_copy_kernel) per step"}
        else:
            # the guide's measured peer copy (770 GB/s per direction), 900 nominal for context
            roof = {"bound": "nvlink", "achieved": round(kernel_gbs, 1), "peak": 770.0, "unit": "GB/s",
                    "frac": round(kernel_gbs / 770.0, 4), "traffic": None,
                    "peak_src": "measured peer copy per direction (B200_PROFILING.md)",
                    "frac_of_nominal_900": round(kernel_gbs / 900.0, 4),
                    "per_launch_bytes": pb}
        extra["roofline"] = roof
        if peer_tune is not None:
            extra["peer_autotune"] = peer_tune
        if a2a is not None or scen_error is not None:
            extra["scenarios"] = {"c5_all_to_all": a2a, "c5_compaction_all_ranks": compaction,
                                  "c3_peer_interference": peer_interf}
            if scen_error is not None:
                extra["scenarios"]["error"] = scen_error
        if world == 1 and not args.no_cpu_baseline:
            # the cpu_baseline leg: the oracle timed on the host cores, and (outside every
            # timed region) the oracle's sampled check of this run's GPU output
            extra["cpu_baseline"] = cpu_baseline(case)
            extra["cpu_baseline"]["parity_check_of_this_run"] = parity_sample(wk, case, src, dst, lo, hi)
        if world == 1 and args.scenarios:
            del src, dst
            torch.cuda.empty_cache()
            extra["scenarios"] = run_scenarios(wk, local, peaks)
        line = {
            "metric": METRIC, "value": round(value, 2), "unit": "GB/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_step, 4),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": "u8", "data": "synthetic",
            "config": {"workload": workload_name(args, case),
                       "payload_gib_per_pair": round(pb / GiB, 3),
                       "placement": "same GPU" if world == 1 else (
                           "pairs 2k->2k+1 over NVLink, " + ("push: the prefill GPU stores into the peer pool"
                                                              if mode["v"] == "push" else
                                                              "pull: the decode GPU loads from the peer pool")),
                       "l2": "inputs >> 126 MB L2 (no flush needed)",
                       "parallelism": f"{n_movers} independent mover(s)", "seed_offset": args.seed},
            "e2e": {"value": round(e2e_value, 2), "unit": "GB/s",
                    "h2d_bytes_per_step": int(8 * case.n), "d2h_bytes_per_step": int(4 * sh.n_layers)},
            "gpu_launches": int(launches),
            "step_ms_rank0": {"p10": round(float(np.percentile(step_ms, 10)), 4),
                              "p50": round(float(np.percentile(step_ms, 50)), 4),
                              "p90": round(float(np.percentile(step_ms, 90)), 4)},
            "clocks": clk_timed,
            # the paper's only migration number, as context (A800, not a target): one
            # 2048-token OPT-13B request = 1.5625 GiB, "~65 ms" over PCIe Gen4 x16
            "paper_context": {
                "p120_request_gib": 1.5625, "p120_pcie_gen4_ms": 65.0, "p120_implied_gbs": 25.8,
                "same_request_ms_at_this_rate": round(1.5625 * GiB / (value / n_movers * 1e6), 3),
                "same_request_ms_at_nvlink5_770gbs": round(1.5625 * GiB / 770e6, 3)},
            **extra,
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


def traffic_from_profiles(cfg: str):
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if not os.path.exists(p):
        return None
    try:
        return json.load(open(p)).get(cfg, {}).get("dram_bytes_per_launch")
    except Exception:
        return None


def workload_name(args, case) -> str:
    """config.workload of both arms (the wind_kv line and --impl reference)."""
    sh = case.shape
    return (f"{args.config} {sh.name} KV: {case.n} blocks of {case.lengths.size} "
            f"requests ({LENGTH_MIX.get(args.config, '')}), {args.variant} tables, "
            f"prefill pool -> decode pool, layers 0-{sh.n_layers - 1}")


def run_reference(args) -> None:
    """--impl reference: the CPU oracle as it stands on this host's cores, rank 0 only."""
    rank = int(os.environ.get("RANK", 0))
    if rank != 0:
        return
    import oracle as O
    from windgen import migration_case
    case = migration_case(args.config, variant=args.variant, seed_offset=args.seed)
    sh = case.shape
    n = min(64, case.n)  # bounded sample per step
    nb = math.ceil(1.1 * n)
    g = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nb)
    src = np.ones(g.pool_bytes, np.uint8)
    dst = np.zeros(g.pool_bytes, np.uint8)
    sbt = np.random.default_rng(1).permutation(nb)[:n].astype(np.int32)
    dbt = np.random.default_rng(2).permutation(nb)[:n].astype(np.int32)
    T = O.hw_threads()
    for _ in range(args.warmup):
        O.migrate_mt(src, g, sbt, dst, g, dbt, 0, sh.n_layers, T)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        assert O.migrate_mt(src, g, sbt, dst, g, dbt, 0, sh.n_layers, T) == O.OK
    el = time.perf_counter() - t0
    pb = payload_bytes(n, sh.n_layers, sh.chunk_bytes)
    v = pb * args.steps / el / 1e9
    sample = f"{n} of {case.n} {args.config} blocks ({pb / GiB:.2f} GiB payload) per step"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": round(v, 3), "unit": "GB/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(el / args.steps * 1e3, 3), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": workload_name(args, case), "sample": "oracle on host cores, bounded sample: " + sample},
        "cpu_baseline": {"value": round(v, 3), "unit": "GB/s", "cores": T, "kind": "oracle",
                         "sample": sample},
        "e2e": {"value": round(v, 3), "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="wind_kv", choices=["wind_kv", "reference"])
    ap.add_argument("--config", default="C2")
    ap.add_argument("--variant", default="shuffled", choices=["shuffled", "sequential"])
    ap.add_argument("--seed", type=int, default=0,
                    help="offset of the config's length / slot / content seeds (0 = the S§8(d) seeds)")
    ap.add_argument("--scenarios", dest="scenarios", action="store_true", default=True)
    ap.add_argument("--no-scenarios", dest="scenarios", action="store_false")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-peer-interference", dest="peer_interference", action="store_false", default=True,
                    help="N > 1: skip the decode-step victims next to the NVLink pushes (~40 GB per rank)")
    ap.add_argument("--a2a-scale", type=float, default=1.0,
                    help="request-count scale of the N>1 all-to-all scenario (C5 = 1.0)")
    args = ap.parse_args()
    if args.warmup < 3:
        raise SystemExit("--warmup must be >= 3")
    if args.impl == "reference":
        run_reference(args)
    else:
        run_gpu(args)


if __name__ == "__main__":
    main()
