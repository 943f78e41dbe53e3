"""GPU: ownership of the per-op arrival-counter slots (include/wind_kv.h "Conventions";
wind_kv_internal.h kEagerSlots).

An op counts its CTAs' arrivals per layer in a counter slot and publishes a layer when the
count completes (A5).  A slot must never be shared by two ops that execute at the
same time.  Round 1-2 handed slots out round robin at enqueue, so an op that stayed pending
for long — a stepped migration waiting on decode steps, an op queued behind a
layer_wait — had its slot handed to the 512th op enqueued after it on another stream.
These tests hold such an op pending while hundreds of ops run elsewhere, and fill every
slot with pending ops, then compare every byte and flag with the oracle.

The gates are host-mapped words (a host pool's layer flags) released by a CPU store, with
a watchdog thread that releases them anyway: a blocked stream can never hang the suite."""
import ctypes as ct
import threading
import time

import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
from rawstreams import raw_streams

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


class HostGate:
    """A uint32 in mapped pinned memory (layer 0 flag of a 1-layer host pool): streams wait
    on it on the GPU (cuStreamWaitValue32), the CPU releases them with a plain store."""

    def __init__(self, watchdog_s: float):
        self.pool = wk.Pool(1, 1, 64, 16, 2, 1, loc="host")
        self.word = ct.c_uint32.from_address(self.pool.flags_ptr)
        self.word.value = 0
        self._stop = threading.Event()
        self._th = threading.Thread(target=self._watch, args=(watchdog_s,), daemon=True)
        self._th.start()

    def _watch(self, s):
        if not self._stop.wait(s):
            self.word.value = 1 << 20  # the test hung: release every waiter

    def set(self, v: int) -> None:
        self.word.value = v

    def close(self) -> None:
        self.word.value = 1 << 20
        self._stop.set()


def geom(L, H, d, bs, eb, nb):
    return O.Geom(0, L, H, d, bs, eb, nb)


def test_pending_stepped_op_keeps_its_counter_slot():
    """A stepped op (slices released by a host-driven step counter) runs its first slice and
    then waits; meanwhile 700 ops over the same layers run to completion on another stream.
    The stepped op keeps its slot: after its remaining slices both destinations equal the
    oracle and every flag counts its ops (1 and 700)."""
    L, H, d, bs, eb = 6, 8, 128, 16, 2  # 32 KiB chunks
    nb, n = 64, 48
    rng = np.random.default_rng(31)
    src = wk.Pool(L, H, d, bs, eb, nb)
    dst = wk.Pool(L, H, d, bs, eb, nb)
    s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    d0 = rng.integers(0, 256, dst.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s0))
    dst.tensor().copy_(torch.from_numpy(d0))
    sbt = rng.permutation(nb)[:n].astype(np.int32)
    dbt = rng.permutation(nb)[:n].astype(np.int32)
    ts, td = torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV)
    osrc = wk.Pool(L, H, d, bs, eb, 16)
    odst = wk.Pool(L, H, d, bs, eb, 16)
    o0 = rng.integers(0, 256, osrc.nbytes, dtype=np.uint8)
    osrc.tensor().copy_(torch.from_numpy(o0))
    odst.tensor().zero_()
    obt_s = np.array([3, 9, 1, 14], np.int32)
    obt_d = np.array([0, 5, 6, 11], np.int32)
    tos, tod = torch.as_tensor(obt_s, device=DEV), torch.as_tensor(obt_d, device=DEV)
    mig, other = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
    torch.cuda.synchronize()
    gate = HostGate(watchdog_s=60)
    try:
        n0 = wk.launch_count()
        payload = 2 * L * n * src.chunk_bytes
        wk.migrate_stepped(src, ts, dst, td, gate.pool.flags_ptr, first_step=1,
                           bytes_per_step=payload // 4 + 1, stream=mig)
        slices = wk.launch_count() - n0
        assert slices >= 4
        gate.set(1)  # slice 0 runs, the rest wait for steps 2, 3, ...
        time.sleep(0.05)
        for _ in range(700):
            wk.migrate(osrc, tos, odst, tod, stream=other)
        other.synchronize()
        assert not mig.query(), "the stepped op should still be waiting for step 2"
        gate.set(slices)
        mig.synchronize()
    finally:
        gate.close()
        torch.cuda.synchronize()
    want = d0.copy()
    assert O.migrate(s0, geom(L, H, d, bs, eb, nb), sbt, want, geom(L, H, d, bs, eb, nb), dbt, 0, L) == O.OK
    np.testing.assert_array_equal(dst.tensor().cpu().numpy(), want)
    assert [dst.layer_count(l) for l in range(L)] == [1] * L
    owant = np.zeros(odst.nbytes, np.uint8)
    assert O.migrate(o0, geom(L, H, d, bs, eb, 16), obt_s, owant, geom(L, H, d, bs, eb, 16), obt_d, 0, L) == O.OK
    np.testing.assert_array_equal(odst.tensor().cpu().numpy(), owant)
    assert [odst.layer_count(l) for l in range(L)] == [700] * L


def test_counter_slots_exhaust_cleanly_and_recover():
    """512 streams each hold a pending op (queued behind a host gate): an op on a 513th
    stream is UNSUPPORTED with nothing enqueued, while a held stream may still queue more
    (its ops share its slot in stream order).  After the gate opens every destination
    equals the oracle and the 513th stream's op goes through."""
    L, H, d, bs, eb = 2, 1, 64, 16, 2  # 2 KiB chunks
    rng = np.random.default_rng(32)
    src = wk.Pool(L, H, d, bs, eb, 8)
    s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s0))
    k = 512
    dsts = [wk.Pool(L, H, d, bs, eb, 8) for _ in range(k + 1)]
    for p in dsts:
        p.tensor().zero_()
    sbt = np.array([7, 2, 5, 0], np.int32)
    dbt = np.array([1, 3, 4, 6], np.int32)
    ts, td = torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV)
    streams = raw_streams(k + 1)  # distinct CUDA streams (torch recycles 32)
    torch.cuda.synchronize()  # every earlier op of the session is done: all slots free
    gate = HostGate(watchdog_s=90)
    try:
        for i in range(k):
            wk.layer_wait(gate.pool, 0, 1, stream=streams[i].handle)
            wk.migrate(src, ts, dsts[i], td, stream=streams[i].handle)
        n0 = wk.launch_count()
        with pytest.raises(wk.WindKVError) as e:
            wk.migrate(src, ts, dsts[k], td, stream=streams[k].handle)
        assert e.value.status == -10 and "counter-slot" in wk.last_error()
        assert wk.launch_count() == n0 and dsts[k].layer_ticket() == 0
        wk.migrate(src, ts, dsts[0], td, layer_lo=1, layer_hi=2, stream=streams[0].handle)  # same stream: OK
        gate.set(1)
        for st in streams[:k]:
            st.synchronize()
    finally:
        gate.close()
        torch.cuda.synchronize()
    wk.migrate(src, ts, dsts[k], td, stream=streams[k].handle)  # slots are free again
    torch.cuda.synchronize()
    for st in streams:
        st.destroy()
    want = np.zeros(src.nbytes, np.uint8)
    g = geom(L, H, d, bs, eb, 8)
    assert O.migrate(s0, g, sbt, want, g, dbt, 0, L) == O.OK
    for i, p in enumerate(dsts):
        np.testing.assert_array_equal(p.tensor().cpu().numpy(), want)
        assert [p.layer_count(l) for l in range(L)] == ([2, 2] if i == 0 else [1, 1])


def test_captured_ops_use_their_own_slots_and_replay_while_eager_ops_run():
    """A captured op (graph slot ring) replayed on one stream while eager ops run on
    another: both destinations equal the oracle, flags count every replay and op."""
    L, H, d, bs, eb = 4, 2, 64, 16, 2
    rng = np.random.default_rng(33)
    src = wk.Pool(L, H, d, bs, eb, 32)
    s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s0))
    a, b = wk.Pool(L, H, d, bs, eb, 32), wk.Pool(L, H, d, bs, eb, 32)
    a.tensor().zero_()
    b.tensor().zero_()
    sbt = rng.permutation(32)[:20].astype(np.int32)
    dbt = rng.permutation(32)[:20].astype(np.int32)
    ts, td = torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV)
    cap, eager = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
    torch.cuda.synchronize()
    graph = torch.cuda.CUDAGraph()
    with torch.cuda.graph(graph, stream=cap):
        wk.migrate(src, ts, a, td, stream=cap)
    torch.cuda.synchronize()
    for _ in range(50):
        with torch.cuda.stream(cap):
            graph.replay()
        wk.migrate(src, ts, b, td, stream=eager)
    torch.cuda.synchronize()
    want = np.zeros(src.nbytes, np.uint8)
    g = geom(L, H, d, bs, eb, 32)
    assert O.migrate(s0, g, sbt, want, g, dbt, 0, L) == O.OK
    for p in (a, b):
        np.testing.assert_array_equal(p.tensor().cpu().numpy(), want)
        assert [p.layer_count(l) for l in range(L)] == [50] * L


def test_debug_table_checks_on_two_streams_do_not_share_scratch():
    """Debug pools run a device-side table check (count kernel + judge kernel over a scratch
    array) before the copy.  Two valid debug ops on two streams at the same time use the
    scratch of their own counter slots: no false DUP_DST / ALIAS, and both copies land."""
    L, H, d, bs, eb = 1, 1, 8, 16, 2  # 256-byte chunks: the table check dominates
    nb, n = 200_000, 150_000
    rng = np.random.default_rng(34)
    src = wk.Pool(L, H, d, bs, eb, nb, debug=True)
    s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s0))
    dsts = [wk.Pool(L, H, d, bs, eb, nb, debug=True) for _ in range(2)]
    for p in dsts:
        p.tensor().zero_()
    tabs = []
    for _ in range(2):
        sbt = rng.permutation(nb)[:n].astype(np.int32)
        dbt = rng.permutation(nb)[:n].astype(np.int32)
        tabs.append((sbt, dbt, torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV)))
    streams = [torch.cuda.Stream(DEV) for _ in range(2)]
    torch.cuda.synchronize()
    for _ in range(10):
        for p, (_, _, ts, td), st in zip(dsts, tabs, streams):
            wk.migrate(src, ts, p, td, stream=st)
    torch.cuda.synchronize()
    for p in dsts:
        wk.check_device_error(p)  # raises DEVICE_CHECK on a (false) table error
    g = geom(L, H, d, bs, eb, nb)
    for p, (sbt, dbt, _, _) in zip(dsts, tabs):
        want = np.zeros(p.nbytes, np.uint8)
        assert O.migrate(s0, g, sbt, want, g, dbt, 0, L) == O.OK
        np.testing.assert_array_equal(p.tensor().cpu().numpy(), want)
        assert p.layer_count(0) == 10


def test_ops_into_one_host_pool_from_two_streams_are_serialised():
    """A host pool's flags are bumped by a plain read-modify-write over PCIe, so ops INTO it
    must not overlap.  Stream A's swap_out waits behind a host gate; stream B's swap_out into
    the same host pool (other host slots) must wait for it — B is still pending while A is
    held — then both land: host pool == oracle, every flag == 2."""
    L, H, d, bs, eb = 4, 2, 64, 16, 2
    rng = np.random.default_rng(35)
    dev = wk.Pool(L, H, d, bs, eb, 32)
    s0 = rng.integers(0, 256, dev.nbytes, dtype=np.uint8)
    dev.tensor().copy_(torch.from_numpy(s0))
    host = wk.Pool(L, H, d, bs, eb, 32, loc="host")
    host.tensor().zero_()
    a_dev, a_host = np.array([4, 9, 1], np.int32), np.array([0, 1, 2], np.int32)
    b_dev, b_host = np.array([30, 2], np.int32), np.array([10, 11], np.int32)
    # the tables are borrowed until the ops complete: keep them alive
    ta_dev, ta_host, tb_dev, tb_host = (torch.as_tensor(x, device=DEV) for x in (a_dev, a_host, b_dev, b_host))
    A, B = raw_streams(2)
    torch.cuda.synchronize()
    gate = HostGate(watchdog_s=60)
    try:
        wk.layer_wait(gate.pool, 0, 1, stream=A.handle)
        wk.swap_out(dev, ta_dev, host, ta_host, stream=A.handle)
        wk.swap_out(dev, tb_dev, host, tb_host, stream=B.handle)
        time.sleep(0.05)
        assert not B.query(), "an op into the host pool overtook a pending one from another stream"
        gate.set(1)
        A.synchronize()
        B.synchronize()
    finally:
        gate.close()
        torch.cuda.synchronize()
    want = np.zeros(host.nbytes, np.uint8)
    g = geom(L, H, d, bs, eb, 32)
    assert O.migrate(s0, g, a_dev, want, g, a_host, 0, L) == O.OK
    assert O.migrate(s0, g, b_dev, want, g, b_host, 0, L) == O.OK
    np.testing.assert_array_equal(host.tensor().cpu().numpy(), want)
    assert [host.layer_count(l) for l in range(L)] == [2] * L
    for s in (A, B):
        s.destroy()


def test_many_swap_outs_into_one_host_pool_from_four_streams():
    """Four streams each enqueue 30 small swap_outs into one host pool (disjoint host slots)
    at once: no flag increment is lost (every flag == 120) and the pool equals the oracle."""
    L, H, d, bs, eb = 3, 1, 64, 16, 2
    rng = np.random.default_rng(36)
    dev = wk.Pool(L, H, d, bs, eb, 64)
    s0 = rng.integers(0, 256, dev.nbytes, dtype=np.uint8)
    dev.tensor().copy_(torch.from_numpy(s0))
    host = wk.Pool(L, H, d, bs, eb, 4 * 30, loc="host")
    host.tensor().zero_()
    streams = raw_streams(4)
    ops = []
    for k in range(4):
        for i in range(30):
            ops.append((k, np.array([rng.integers(0, 64)], np.int32), np.array([k * 30 + i], np.int32)))
    tabs = [(k, torch.as_tensor(sd, device=DEV), torch.as_tensor(hd, device=DEV), sd, hd) for k, sd, hd in ops]
    torch.cuda.synchronize()
    for i in range(30):  # interleaved across the four streams
        for k in range(4):
            _, tsd, thd, _, _ = tabs[k * 30 + i]
            wk.swap_out(dev, tsd, host, thd, stream=streams[k].handle)
    torch.cuda.synchronize()
    want = np.zeros(host.nbytes, np.uint8)
    gd, gh = geom(L, H, d, bs, eb, 64), geom(L, H, d, bs, eb, 120)
    for _, _, _, sd, hd in tabs:
        assert O.migrate(s0, gd, sd, want, gh, hd, 0, L) == O.OK
    np.testing.assert_array_equal(host.tensor().cpu().numpy(), want)
    assert [host.layer_count(l) for l in range(L)] == [120] * L
    for s in streams:
        s.destroy()


def test_staged_swaps_on_one_host_pool_from_four_host_threads():
    """The staged copy-engine path (kernel 4) reuses a host pool's staging buffers and
    events; ops on one host pool are enqueued under the pool's lock, so four host threads
    may issue staged swap_ins from one host pool at once (each into its own device pool, on
    its own stream): every device pool equals the oracle, every flag == 3."""
    L, H, d, bs, eb = 4, 4, 64, 16, 2
    rng = np.random.default_rng(37)
    host = wk.Pool(L, H, d, bs, eb, 64, loc="host")
    h0 = rng.integers(0, 256, host.nbytes, dtype=np.uint8)
    host.tensor().copy_(torch.from_numpy(h0))
    devs = [wk.Pool(L, H, d, bs, eb, 48) for _ in range(4)]
    for p in devs:
        p.tensor().zero_()
    plans = []
    for k in range(4):
        ops = []
        for _ in range(3):
            hb = rng.permutation(64)[:10].astype(np.int32)   # host side: read on the CPU (pinned)
            db = rng.permutation(48)[:10].astype(np.int32)
            ops.append((hb, db, torch.as_tensor(hb).pin_memory(), torch.as_tensor(db, device=DEV)))
        plans.append((devs[k], raw_streams(1)[0], ops))
    saved = wk.get_tuning(wk.PATH_HOST)
    wk.set_tuning(wk.PATH_HOST, kernel=wk.KERNEL_STAGED)
    errors = []
    torch.cuda.synchronize()

    def worker(dev, stream, ops):
        try:
            for _, _, thb, tdb in ops:
                wk.swap_in(host, thb, dev, tdb, stream=stream.handle)
        except Exception as e:  # noqa: BLE001 — reported below
            errors.append(e)
    try:
        threads = [threading.Thread(target=worker, args=pl) for pl in plans]
        for th in threads:
            th.start()
        for th in threads:
            th.join()
        torch.cuda.synchronize()
    finally:
        wk.set_tuning(wk.PATH_HOST, **saved)
    assert not errors, errors
    g_h, g_d = geom(L, H, d, bs, eb, 64), geom(L, H, d, bs, eb, 48)
    for dev, stream, ops in plans:
        want = np.zeros(dev.nbytes, np.uint8)
        for hb, db, _, _ in ops:
            assert O.migrate(h0, g_h, hb, want, g_d, db, 0, L) == O.OK
        np.testing.assert_array_equal(dev.tensor().cpu().numpy(), want)
        assert [dev.layer_count(l) for l in range(L)] == [3] * L
        stream.destroy()


def test_two_streams_of_ops_into_one_device_pool():
    """R21: concurrent ops into one destination pool with disjoint destination slots.  Two
    streams enqueue 100 ops each (random layer ranges, interleaved) into one device pool:
    the pool equals the oracle (the ops commute: disjoint slots) and every layer flag counts
    all 200 ops (an op bumps every destination layer once, R23)."""
    L, H, d, bs, eb = 6, 2, 64, 16, 2
    rng = np.random.default_rng(38)
    src = wk.Pool(L, H, d, bs, eb, 64)
    s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s0))
    dst = wk.Pool(L, H, d, bs, eb, 400)
    dst.tensor().zero_()
    A, B = raw_streams(2)
    ops = []
    slots = rng.permutation(400).astype(np.int32)
    for i in range(200):
        sb = rng.permutation(64)[:2].astype(np.int32)
        db = slots[2 * i:2 * i + 2].copy()
        lo = int(rng.integers(0, L))
        hi = int(rng.integers(lo + 1, L + 1))
        ops.append((sb, db, lo, hi, torch.as_tensor(sb, device=DEV), torch.as_tensor(db, device=DEV)))
    torch.cuda.synchronize()
    for i, (_, _, lo, hi, ts, td) in enumerate(ops):
        wk.migrate(src, ts, dst, td, layer_lo=lo, layer_hi=hi, stream=(A if i % 2 else B).handle)
    torch.cuda.synchronize()
    want = np.zeros(dst.nbytes, np.uint8)
    gs, gd = geom(L, H, d, bs, eb, 64), geom(L, H, d, bs, eb, 400)
    for sb, db, lo, hi, _, _ in ops:
        assert O.migrate(s0, gs, sb, want, gd, db, lo, hi) == O.OK
    np.testing.assert_array_equal(dst.tensor().cpu().numpy(), want)
    assert dst.layer_ticket() == 200 and [dst.layer_count(l) for l in range(L)] == [200] * L
    for s in (A, B):
        s.destroy()


def test_stepped_op_across_the_step_counter_wrap():
    """wind_kv.h: slice k of a stepped op is released when the step counter reaches
    first_step + k, 'wrap-safe' (cuStreamWaitValue32 GEQ compares (int32)(*addr - value)).
    Steps 2^32-2, 2^32-1, 0, 1, ... straddle the uint32 wrap: slices stay blocked until
    their step, then all land (whole pool == oracle, one flag bump per layer).  The gate is a
    host-mapped word; its watchdog alternates two release values so a wrong comparison
    cannot hang the suite."""
    L, H, d, bs, eb = 8, 8, 128, 16, 2  # 32 KiB chunks
    nb, n = 48, 40
    rng = np.random.default_rng(39)
    src, dst = wk.Pool(L, H, d, bs, eb, nb), wk.Pool(L, H, d, bs, eb, nb)
    s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    d0 = rng.integers(0, 256, dst.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s0))
    dst.tensor().copy_(torch.from_numpy(d0))
    sbt = rng.permutation(nb)[:n].astype(np.int32)
    dbt = rng.permutation(nb)[:n].astype(np.int32)
    ts, td = torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV)
    word_pool = wk.Pool(1, 1, 64, 16, 2, 1, loc="host")
    word = ct.c_uint32.from_address(word_pool.flags_ptr)
    first = (1 << 32) - 2
    word.value = first - 1
    stop = threading.Event()

    def watchdog():
        if stop.wait(30):
            return
        for i in range(400):  # release under either comparison, alternately
            word.value = 0xFFFFFFFF if i % 2 else (1 << 20)
            time.sleep(0.025)
    wd = threading.Thread(target=watchdog, daemon=True)
    wd.start()
    mig = raw_streams(1)[0]
    torch.cuda.synchronize()
    try:
        n0 = wk.launch_count()
        payload = 2 * L * n * src.chunk_bytes
        wk.migrate_stepped(src, ts, dst, td, word_pool.flags_ptr, first_step=first,
                           bytes_per_step=payload // 6 + 1, stream=mig.handle)
        slices = wk.launch_count() - n0
        assert slices >= 4
        time.sleep(0.05)
        assert not mig.query(), "released before its first step"
        for k in range(slices - 1):  # steps first .. first + slices - 2 (crossing 2^32)
            word.value = (first + k) & 0xFFFFFFFF
            time.sleep(0.05)
            assert not mig.query(), f"last slice released at step {k} of {slices}"
        word.value = (first + slices - 1) & 0xFFFFFFFF
        t_end = time.time() + 10
        while not mig.query() and time.time() < t_end:
            time.sleep(0.01)
        assert mig.query(), "the last slice was not released at its step"
    finally:
        # whatever happened above, release every slice under either comparison before
        # anything synchronises (bounded), then stop the watchdog
        t_end = time.time() + 20
        i = 0
        while not mig.query() and time.time() < t_end:
            word.value = 0xFFFFFFFF if i % 2 else (1 << 20)
            i += 1
            time.sleep(0.025)
        stop.set()
        torch.cuda.synchronize()
    want = d0.copy()
    g = geom(L, H, d, bs, eb, nb)
    assert O.migrate(s0, g, sbt, want, g, dbt, 0, L) == O.OK
    np.testing.assert_array_equal(dst.tensor().cpu().numpy(), want)
    assert [dst.layer_count(l) for l in range(L)] == [1] * L
    mig.destroy()
