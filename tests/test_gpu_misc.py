"""GPU: CUDA-graph capture of the ops, external pool bases, and launch accounting."""
import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
from windgen import migration_case, KVShape

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def geom(p):
    d = p.desc
    return O.Geom(d.first_layer, d.n_layers, d.n_kv_heads, d.head_dim, d.block_size, d.elem_bytes,
                  d.n_blocks)


def test_migrate_is_graph_capturable():
    """wind_kv.h: ops never allocate or synchronise, so they can be captured in a CUDA
    graph and replayed (the layer flags count every replay)."""
    case = migration_case("C1", scale=0.5)
    sh = case.shape
    src = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, case.nb_src)
    dst = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, case.nb_dst)
    rng = np.random.default_rng(0)
    s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    d0 = rng.integers(0, 256, dst.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s0))
    dst.tensor().copy_(torch.from_numpy(d0))
    ts = torch.as_tensor(case.src_bt, device=DEV)
    td = torch.as_tensor(case.dst_bt, device=DEV)
    s = torch.cuda.Stream(DEV)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        wk.migrate(src, ts, dst, td, layer_lo=2, layer_hi=9, stream=s)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(dst.tensor().cpu().numpy(), d0)  # capture ran nothing
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    want = d0.copy()
    assert O.migrate(s0, geom(src), case.src_bt, want, geom(dst), case.dst_bt, 2, 9) == O.OK
    np.testing.assert_array_equal(dst.tensor().cpu().numpy(), want)
    assert all(dst.layer_count(l) == 3 for l in range(sh.n_layers))


def test_external_base_pools():
    """Pools over caller memory (torch allocations): used in place, never freed by the
    library; a misaligned base is INVALID_ARG."""
    sh = KVShape("t", 2, 4, 64, 2)
    nb = 30
    nbytes = sh.n_layers * 2 * nb * sh.chunk_bytes
    buf_s = torch.randint(0, 256, (nbytes,), dtype=torch.uint8, device=DEV)
    buf_d = torch.randint(0, 256, (nbytes + 16,), dtype=torch.uint8, device=DEV)
    src = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nb,
                  external_base=buf_s.data_ptr())
    with pytest.raises(wk.WindKVError) as e:
        wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nb,
                external_base=buf_d.data_ptr() + 8)
    assert e.value.status == -1
    dst = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nb,
                  external_base=buf_d.data_ptr() + 16)
    assert src.base == buf_s.data_ptr() and dst.base == buf_d.data_ptr() + 16
    s0, d0 = buf_s.cpu().numpy().copy(), buf_d[16:].cpu().numpy().copy()
    sbt, dbt = np.array([3, 9, 29, 0], np.int32), np.array([1, 2, 3, 28], np.int32)
    wk.migrate(src, torch.as_tensor(sbt, device=DEV), dst, torch.as_tensor(dbt, device=DEV))
    torch.cuda.synchronize()
    want = d0.copy()
    g = O.Geom(0, 2, 4, 64, 16, 2, nb)
    assert O.migrate(s0, g, sbt, want, g, dbt, 0, 2) == O.OK
    np.testing.assert_array_equal(buf_d[16:].cpu().numpy(), want)
    src.destroy()
    dst.destroy()
    assert buf_s.sum().item() >= 0  # caller memory still valid after destroy


def test_launch_count_one_kernel_per_op():
    sh = KVShape("t", 2, 4, 64, 2)
    a = wk.Pool(2, 4, 64, 16, 2, 20)
    b = wk.Pool(2, 4, 64, 16, 2, 20)
    t = torch.arange(10, dtype=torch.int32, device=DEV)
    n0 = wk.launch_count()
    for _ in range(7):
        wk.migrate(a, t, b, t)
    wk.migrate_batch(a, [(b, t, t)], 0, 2)
    torch.cuda.synchronize()
    assert wk.launch_count() - n0 == 8
    del sh


@pytest.mark.parametrize("max_ctas", [0, 4])
def test_rate_limit_paces_the_copy(max_ctas):
    """wind_kv_tuning.rate_mbps bounds an op's payload rate (interference budget) without
    changing its result: burst pacing (max_ctas 0: full-grid slices between 1-thread pace
    kernels) and the in-kernel pacer (a CTA cap: a small paced grid)."""
    from windgen import SHAPES
    import windgen.cuda as wg
    sh = SHAPES["C2"]
    nb = 300
    src = wk.Pool(4, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
    dst = wk.Pool(4, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
    wg.fill(src.base, src.nbytes, 0, 1, 1)
    wg.fill(dst.base, dst.nbytes, 0, 1, 2)
    sbt = torch.randperm(nb, generator=torch.Generator().manual_seed(0))[:256].to(torch.int32).to(DEV)
    dbt = torch.randperm(nb, generator=torch.Generator().manual_seed(1))[:256].to(torch.int32).to(DEV)
    payload = 2 * 4 * 256 * sh.chunk_bytes  # 320 MiB
    saved = wk.get_tuning(wk.PATH_INTRA)
    s = torch.cuda.Stream(DEV)
    try:
        for rate_gbs in (20, 80):
            wk.set_tuning(wk.PATH_INTRA, **{**saved, "rate_mbps": rate_gbs * 1000, "max_ctas": max_ctas})
            a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            a.record(s)
            n0 = wk.launch_count()
            wk.migrate(src, sbt, dst, dbt, stream=s)
            b.record(s)
            if max_ctas == 0:  # 2 ms of rate budget per burst, a pace kernel before and after each
                bursts = (wk.launch_count() - n0 - 1) // 2
                assert abs(bursts - payload / (rate_gbs * 1e9 * 2e-3)) <= 1.5, bursts
            else:
                assert wk.launch_count() - n0 == 1
            torch.cuda.synchronize()
            got = payload / (a.elapsed_time(b) * 1e6)
            assert 0.75 * rate_gbs < got < 1.1 * rate_gbs, (rate_gbs, got)
    finally:
        wk.set_tuning(wk.PATH_INTRA, **saved)
    S = src.tensor().view(4, 2, nb, -1)
    D = dst.tensor().view(4, 2, nb, -1)
    assert torch.equal(D[:, :, dbt.long()], S[:, :, sbt.long()])


def test_burst_paced_op_flags_and_parity():
    """A burst-paced op (rate limit, no CTA cap) is many launches on ONE arrival-counter slot:
    a consumer stream waits on every layer flag and snapshots the layer — each snapshot
    already holds the oracle's bytes — the whole pool equals the oracle, every flag moves
    exactly once, and a layer window leaves the other layers' bytes alone."""
    import oracle as O
    from windgen import SHAPES
    sh = SHAPES["C2"]
    L, nb, n = 8, 200, 150
    src = wk.Pool(L, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
    dst = wk.Pool(L, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
    rng = np.random.default_rng(5)
    s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    d0 = rng.integers(0, 256, dst.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s0))
    dst.tensor().copy_(torch.from_numpy(d0))
    sbt = rng.permutation(nb)[:n].astype(np.int32)
    dbt = rng.permutation(nb)[:n].astype(np.int32)
    ts, td = torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV)
    want = d0.copy()
    g = O.Geom(0, L, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
    assert O.migrate(s0, g, sbt, want, g, dbt, 1, 7) == O.OK
    plane = nb * sh.chunk_bytes
    view = dst.tensor()
    snaps = torch.empty(L, 2 * plane, dtype=torch.uint8, device=DEV)
    s, cons = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
    torch.cuda.synchronize()
    n0 = wk.launch_count()
    # 2 x 6 layers x 150 blocks x 160 KiB = 281 MiB at 50 GB/s: ~3 bursts of 100 MB
    wk.migrate_ex(src, ts, dst, td, wk.tuning(rate_mbps=50_000, max_ctas=0),
                  layer_lo=1, layer_hi=7, stream=s)
    launches = wk.launch_count() - n0
    assert launches >= 5 and launches % 2 == 1  # 1 + 2 x bursts
    t = dst.layer_ticket()
    with torch.cuda.stream(cons):
        for l in range(L):
            wk.layer_wait(dst, l, t, stream=cons)
            snaps[l].copy_(view[l * 2 * plane:(l + 1) * 2 * plane])
    torch.cuda.synchronize()
    np.testing.assert_array_equal(snaps.cpu().numpy().reshape(-1), want)
    np.testing.assert_array_equal(view.cpu().numpy(), want)
    assert [dst.layer_count(l) for l in range(L)] == [1] * L


def test_plain_c_abi_user():
    """examples/c_abi_example.c drives the library through the C ABI alone."""
    import os
    import subprocess
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    exe = os.path.join(root, "examples", "c_abi_example")
    if not os.path.exists(exe):
        import __graft_entry__
        __graft_entry__.build_c_example()
    out = subprocess.run([exe], capture_output=True, text=True, timeout=300)
    assert out.returncode == 0, out.stderr
    assert "c_abi_example OK" in out.stdout


def test_many_concurrent_ops_across_streams():
    """200 ops enqueued at once on 200 distinct CUDA streams (each into its own destination
    pool), plus a 40-op layer-streamed sequence on one stream: every pending op holds its
    own arrival-counter slot; all data byte-exact vs the oracle, every flag == its ticket."""
    import oracle as O
    from rawstreams import raw_streams
    raws = raw_streams(200)
    L, H, d, bs, eb = 4, 2, 64, 16, 2
    rng = np.random.default_rng(7)
    src = wk.Pool(L, H, d, bs, eb, 64)
    s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s0))
    dsts, jobs = [], []
    for k in range(200):
        p = wk.Pool(L, H, d, bs, eb, 32)
        p.tensor().zero_()
        sbt = rng.permutation(64)[:20].astype(np.int32)
        dbt = rng.permutation(32)[:20].astype(np.int32)
        dsts.append(p)
        jobs.append((p, raws[k].handle, torch.as_tensor(sbt, device="cuda"),
                     torch.as_tensor(dbt, device="cuda"), sbt, dbt))
    torch.cuda.synchronize()
    for p, st, ts, td, _, _ in jobs:
        wk.migrate(src, ts, p, td, stream=st)
    one = wk.Pool(L, H, d, bs, eb, 32)
    one.tensor().zero_()
    torch.cuda.synchronize()
    st1 = torch.cuda.Stream()
    ts = torch.as_tensor(np.arange(16, dtype=np.int32), device="cuda")
    for rep in range(10):
        for l in range(L):
            wk.migrate(src, ts, one, ts, layer_lo=l, layer_hi=l + 1, stream=st1)
    torch.cuda.synchronize()
    g = lambda nb: O.Geom(0, L, H, d, bs, eb, nb)  # noqa: E731
    for p, _, _, _, sbt, dbt in jobs:
        want = np.zeros(p.nbytes, np.uint8)
        assert O.migrate(s0, g(64), sbt, want, g(32), dbt, 0, L) == O.OK
        np.testing.assert_array_equal(p.tensor().cpu().numpy(), want)
        assert [p.layer_count(l) for l in range(L)] == [1] * L
    assert one.layer_ticket() == 40 and [one.layer_count(l) for l in range(L)] == [40] * L
    for r in raws:
        r.destroy()


def test_ops_enqueued_from_many_host_threads():
    """Four host threads enqueue 40 ops each at the same time (ctypes releases the GIL inside
    the library), each thread into its own destination pools on its own stream, from one
    shared source pool: every destination byte-exact vs the oracle, every ticket and flag
    right (the per-device counter ring, the pools' ticket counters and the tuning table are
    shared state)."""
    import threading
    import oracle as O
    L, H, d, bs, eb = 4, 2, 64, 16, 2
    rng = np.random.default_rng(11)
    src = wk.Pool(L, H, d, bs, eb, 64)
    s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s0))
    plans = []
    for t in range(4):
        pools = [wk.Pool(L, H, d, bs, eb, 24) for _ in range(4)]
        for p in pools:
            p.tensor().zero_()
        ops = []
        for k in range(40):
            sbt = rng.permutation(64)[:12].astype(np.int32)
            dbt = rng.permutation(24)[:12].astype(np.int32)
            lo = int(rng.integers(0, L))
            ops.append((k % 4, torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV),
                        sbt, dbt, lo, lo + 1))
        plans.append((pools, torch.cuda.Stream(DEV), ops))
    torch.cuda.synchronize()
    errors = []

    def worker(pools, stream, ops):
        try:
            for j, ts, td, _, _, lo, hi in ops:
                wk.migrate(src, ts, pools[j], td, layer_lo=lo, layer_hi=hi, stream=stream)
        except Exception as e:  # noqa: BLE001 — reported below
            errors.append(e)
    threads = [threading.Thread(target=worker, args=pl) for pl in plans]
    for th in threads:
        th.start()
    for th in threads:
        th.join()
    torch.cuda.synchronize()
    assert not errors, errors
    g = lambda nb: O.Geom(0, L, H, d, bs, eb, nb)  # noqa: E731
    for pools, _, ops in plans:
        want = [np.zeros(p.nbytes, np.uint8) for p in pools]
        for j, _, _, sbt, dbt, lo, hi in ops:  # one stream per thread: in order
            assert O.migrate(s0, g(64), sbt, want[j], g(24), dbt, lo, hi) == O.OK
        for p, w in zip(pools, want):
            np.testing.assert_array_equal(p.tensor().cpu().numpy(), w)
            assert p.layer_ticket() == 10 and [p.layer_count(l) for l in range(L)] == [10] * L


def test_migrate_stepped_releases_slices_per_step():
    """wind_kv_migrate_stepped: the op is cut into slices released one per consumer step
    (wind_kv_step_signal): nothing moves before the first signal; after enough signals the
    whole pool equals the oracle, every layer flag moved exactly once, one ticket."""
    import time
    import oracle as O
    from windgen import SHAPES
    sh = SHAPES["C2"]
    L, nb, n = 6, 160, 120
    src = wk.Pool(L, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
    dst = wk.Pool(L, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
    rng = np.random.default_rng(9)
    s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    d0 = rng.integers(0, 256, dst.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s0))
    dst.tensor().copy_(torch.from_numpy(d0))
    sbt = rng.permutation(nb)[:n].astype(np.int32)
    dbt = rng.permutation(nb)[:n].astype(np.int32)
    ts, td = torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV)
    counter = torch.zeros(1, dtype=torch.int32, device=DEV)
    mig, dec = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
    payload = 2 * L * n * sh.chunk_bytes  # 225 MiB -> 5 slices of ~48 MB
    torch.cuda.synchronize()
    n0 = wk.launch_count()
    wk.migrate_stepped(src, ts, dst, td, counter, first_step=1, bytes_per_step=payload // 5 + 1, stream=mig)
    slices = wk.launch_count() - n0
    assert 4 <= slices <= 6 and dst.layer_ticket() == 1
    time.sleep(0.05)
    assert not mig.query()  # blocked on step 1
    np.testing.assert_array_equal(dst.tensor().cpu().numpy(), d0)  # nothing moved yet
    for _ in range(slices):
        wk.step_signal(counter, stream=dec)
        dec.synchronize()
    mig.synchronize()
    assert int(counter.item()) == slices
    want = d0.copy()
    g = O.Geom(0, L, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
    assert O.migrate(s0, g, sbt, want, g, dbt, 0, L) == O.OK
    np.testing.assert_array_equal(dst.tensor().cpu().numpy(), want)
    assert [dst.layer_count(l) for l in range(L)] == [1] * L
    # argument errors, nothing enqueued
    n1 = wk.launch_count()
    for bad in (dict(step_counter=0), dict(bytes_per_step=0)):
        kw = dict(step_counter=counter, first_step=1, bytes_per_step=1 << 20)
        kw.update(bad)
        with pytest.raises(wk.WindKVError) as e:
            wk.migrate_stepped(src, ts, dst, td, stream=mig, **kw)
        assert e.value.status == -1
    host = wk.Pool(L, sh.n_kv_heads, sh.head_dim, 16, 2, nb, loc="host")
    with pytest.raises(wk.WindKVError) as e:
        wk.migrate_stepped(src, ts, host, td, counter, 1, 1 << 20, stream=mig)
    assert e.value.status == -10
    assert wk.launch_count() == n1 and dst.layer_ticket() == 1


def test_pool_larger_than_hbm_is_oom_and_recoverable():
    """A device pool larger than the GPU's memory: WIND_ERR_OOM with the requested size in
    the message, nothing leaked, and the next pool creation works (no sticky CUDA error)."""
    free, _ = torch.cuda.mem_get_info()
    nb = int(2 * free // (40 * 2 * 40 * 16 * 128 * 2)) + 1  # 2x the free memory, OPT-13B KV blocks
    with pytest.raises(wk.WindKVError) as e:
        wk.Pool(40, 40, 128, 16, 2, nb)
    assert e.value.status == -9 and "cudaMalloc" in str(e.value)
    p = wk.Pool(2, 2, 64, 16, 2, 4)
    assert p.nbytes == 2 * 2 * 4 * 2 * 16 * 64 * 2
    torch.cuda.synchronize()
