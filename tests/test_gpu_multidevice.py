"""Multi-GPU parity (SURVEY.md §4 "Multi-GPU parity", §8(e)): pools on two (or more)
devices of one process — push (A4, prefill -> decode hand-off, executes on the source
GPU), pull, one-launch all-to-all to several devices (A8), host swaps served by another
GPU's copy engines — and the multi-process CUDA IPC push across devices.

Cross-device tests need as many GPUs as they name and are SKIPPED otherwise (a one-GPU
box would only run the intra-device route and prove nothing about NVLink); when they run
they assert, through wind_kv_route, that the op took the PEER route with system-scope flag
publication.  The one-launch all-to-all also runs with every pool on device 0, asserting
the INTRA route, so its batching logic is covered on any box.  Every result is compared
byte for byte with the CPU oracle over the whole destination pool.
"""
import multiprocessing as mp
import os
import sys

import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
from windgen import KVShape

pytestmark = pytest.mark.gpu
SH = KVShape("t", 4, 8, 128, 2)  # C = 32 KiB
SHAPE_ARGS = (SH.n_layers, SH.n_kv_heads, SH.head_dim, SH.block_size, SH.elem_bytes)


def devices(k: int) -> list:
    """k distinct GPUs, or skip: a cross-device test on fewer GPUs would silently run the
    intra-device route instead of the one it names."""
    n = torch.cuda.device_count()
    if n < k:
        pytest.skip(f"needs {k} GPUs (NVLink peer route), this box has {n}")
    return list(range(k))


def assert_route(src: wk.Pool, dst: wk.Pool, exec_dev: int, path: int) -> None:
    e, p, sys_scope = wk.route(src, dst)
    assert (e, p) == (exec_dev, path), (e, p)
    forced = os.environ.get("WIND_KV_FORCE_SYS_SCOPE") == "1"  # test_gpu_sys_scope.py
    assert sys_scope == (path != wk.PATH_INTRA or forced)


def geom(p: wk.Pool) -> O.Geom:
    d = p.desc
    return O.Geom(d.first_layer, d.n_layers, d.n_kv_heads, d.head_dim, d.block_size, d.elem_bytes,
                  d.n_blocks)


def pool(nb: int, seed: int, device: int, loc="device"):
    p = wk.Pool(*SHAPE_ARGS, nb, loc=loc, device=device)
    host = np.random.default_rng(seed).integers(0, 256, p.nbytes, dtype=np.uint8)
    p.tensor().copy_(torch.from_numpy(host))
    return p, host


def read(p: wk.Pool) -> np.ndarray:
    for d in range(torch.cuda.device_count()):
        torch.cuda.synchronize(d)
    return p.tensor().cpu().numpy().copy()


_KEEP: list = []  # block tables are BORROWED until their op completes (wind_kv.h)


@pytest.fixture(autouse=True)
def keep_tables_alive():
    yield
    for d in range(torch.cuda.device_count()):
        torch.cuda.synchronize(d)
    _KEEP.clear()


def tab(a, device: int) -> torch.Tensor:
    """A device table that stays alive until the test ends: the ops run on side streams, so a
    temporary freed after the call could be reused by the caching allocator (on the default
    stream) while the kernel still reads it."""
    t = torch.as_tensor(np.asarray(a, np.int32), device=torch.device("cuda", device))
    _KEEP.append(t)
    return t


def test_push_then_pull_across_devices():
    """migrate(src on GPU a -> dst on GPU b) runs on a (push, peer stores); the consumer on b
    waits on dst's flags; then migrate(dst on b -> back on a) runs on b (push the other way)."""
    a, b = devices(2)
    rng = np.random.default_rng(1)
    src, s0 = pool(150, 1, a)
    dst, d0 = pool(120, 2, b)
    sbt = rng.permutation(150)[:77].astype(np.int32)
    dbt = rng.permutation(120)[:77].astype(np.int32)
    sa, sb = torch.cuda.Stream(device=a), torch.cuda.Stream(device=b)
    assert_route(src, dst, a, wk.PATH_PEER)
    wk.migrate(src, tab(sbt, a), dst, tab(dbt, a), layer_lo=1, layer_hi=4, stream=sa)
    t = dst.layer_ticket()
    for l in range(4):
        wk.layer_wait(dst, l, t, stream=sb)
    flags = torch.zeros(4, dtype=torch.int32).pin_memory()
    dst.read_flags(flags, stream=sb)
    sb.synchronize()
    assert flags.tolist() == [1, 1, 1, 1]
    want = d0.copy()
    assert O.migrate(s0, geom(src), sbt, want, geom(dst), dbt, 1, 4) == O.OK
    np.testing.assert_array_equal(read(dst), want)
    back, k0 = pool(40, 3, a)
    pbt = np.arange(5, 35, dtype=np.int32)
    assert_route(dst, back, b, wk.PATH_PEER)
    wk.migrate(dst, tab(dbt[:30], b), back, tab(pbt, b), stream=sb)
    want_b = k0.copy()
    assert O.migrate(want, geom(dst), dbt[:30], want_b, geom(back), pbt, 0, 4) == O.OK
    np.testing.assert_array_equal(read(back), want_b)


@pytest.mark.parametrize("placement", ["peer", "same_device"])
def test_all_to_all_one_launch_per_device(placement):
    """A8 from one process: every pool pushes its outgoing blocks to every other pool in ONE
    wind_kv_migrate_batch launch; destination slots are disjoint (the planner's contract);
    every pool is byte-exact afterwards.  "peer": one pool on each of 2-4 GPUs (PEER route,
    skipped on a one-GPU box); "same_device": 4 pools on device 0 (INTRA route)."""
    devs = devices(2) + list(range(2, min(4, torch.cuda.device_count()))) if placement == "peer" \
        else [0] * 4
    G, nb, per = len(devs), 200, 30
    pools = [pool(nb, 10 + g, devs[g]) for g in range(G)]
    before = [h.copy() for _, h in pools]
    after = [h.copy() for _, h in pools]
    rng = np.random.default_rng(5)
    # destination g receives `per` blocks from each other source in disjoint free slots
    free = [rng.permutation(np.arange(nb // 2, nb)) for _ in range(G)]  # upper half: free
    used = [0] * G
    streams = [torch.cuda.Stream(device=d) for d in devs]
    plans = []
    for s in range(G):
        items = []
        for d in range(G):
            if d == s:
                continue
            sb_ = rng.choice(nb // 2, per, replace=False).astype(np.int32)  # live lower half
            db_ = free[d][used[d]:used[d] + per].astype(np.int32)
            used[d] += per
            items.append((d, sb_, db_))
        plans.append(items)
    for s in range(G):
        for d, _, _ in plans[s]:
            assert_route(pools[s][0], pools[d][0], devs[s],
                         wk.PATH_PEER if placement == "peer" else wk.PATH_INTRA)
        wk.migrate_batch(pools[s][0], [(pools[d][0], tab(sb_, devs[s]), tab(db_, devs[s]))
                                       for d, sb_, db_ in plans[s]], 0, SH.n_layers, stream=streams[s])
    for s in range(G):
        for d, sb_, db_ in plans[s]:
            assert O.migrate(before[s], geom(pools[s][0]), sb_, after[d], geom(pools[d][0]), db_,
                             0, SH.n_layers) == O.OK
    for g in range(G):
        np.testing.assert_array_equal(read(pools[g][0]), after[g])
        assert pools[g][0].layer_ticket() == G - 1
        assert [pools[g][0].layer_count(l) for l in range(SH.n_layers)] == [G - 1] * SH.n_layers


@pytest.mark.parametrize("staging_device", ["same", "other"])
def test_swap_from_second_device(staging_device):
    """A device pool on GPU b swaps out to / in from a host pool.  A host pool whose staging
    lives on b can take the opt-in staged copy-engine path; one whose staging lives on another
    GPU only the SM path over mapped memory (the auto choice, which every case here uses).
    Both byte-exact; the op executes on b."""
    a, b = devices(2)
    rng = np.random.default_rng(6)
    dev, d0 = pool(90, 20, b)
    host, h0 = pool(70, 22, b if staging_device == "same" else a, loc="host")
    hpin = torch.as_tensor(rng.permutation(70)[:60].astype(np.int32)).pin_memory()
    dbt = rng.permutation(90)[:60].astype(np.int32)
    sb = torch.cuda.Stream(device=b)
    assert_route(dev, host, b, wk.PATH_HOST)
    n0 = wk.launch_count()
    wk.swap_out(dev, tab(dbt, b), host, hpin, stream=sb)
    sb.synchronize()
    assert wk.launch_count() - n0 == 1  # one SM kernel over mapped memory
    want_h = h0.copy()
    assert O.swap_out(d0, geom(dev), dbt, want_h, geom(host), hpin.numpy()) == O.OK
    np.testing.assert_array_equal(host.tensor().numpy(), want_h)
    dev2, e0 = pool(80, 21, b)
    dbt2 = rng.permutation(80)[:60].astype(np.int32)
    wk.swap_in(host, hpin, dev2, tab(dbt2, b), stream=sb)
    want2 = e0.copy()
    assert O.swap_in(want_h, geom(host), hpin.numpy(), want2, geom(dev2), dbt2) == O.OK
    np.testing.assert_array_equal(read(dev2), want2)


def _owner(q_out, q_in, device, nb, seed):
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import numpy as np2  # noqa
    import torch as t2  # noqa
    import paper_conf_isca_fenghzly025_b200 as wk2
    t2.cuda.set_device(device)
    p = wk2.Pool(*SHAPE_ARGS, nb, device=device)
    init = np2.random.default_rng(seed).integers(0, 256, p.nbytes, dtype=np2.uint8)
    p.tensor().copy_(t2.from_numpy(init))
    t2.cuda.synchronize()
    q_out.put(p.export())
    q_in.get(timeout=300)  # the importer's push is complete
    t2.cuda.synchronize()
    q_out.put((p.tensor().cpu().numpy(), [p.layer_count(l) for l in range(SH.n_layers)]))
    q_in.get(timeout=300)


def test_ipc_push_across_devices():
    """Multi-process (one process per GPU, as under torchrun): the decode process owns a pool
    on GPU b and exports it; this process imports it on GPU a and pushes into it."""
    a, b = devices(2)
    ctx = mp.get_context("spawn")
    q_out, q_in = ctx.Queue(), ctx.Queue()
    proc = ctx.Process(target=_owner, args=(q_out, q_in, b, 100, 31))
    proc.start()
    try:
        remote = wk.Pool.import_(q_out.get(timeout=300), a)
        src, s0 = pool(130, 30, a)
        assert_route(src, remote, a, wk.PATH_PEER)
        rng = np.random.default_rng(7)
        sbt = rng.permutation(130)[:64].astype(np.int32)
        dbt = rng.permutation(100)[:64].astype(np.int32)
        sa = torch.cuda.Stream(device=a)
        wk.migrate(src, tab(sbt, a), remote, tab(dbt, a), stream=sa)
        sa.synchronize()
        q_in.put("done")
        got, counts = q_out.get(timeout=300)
        want = np.random.default_rng(31).integers(0, 256, got.size, dtype=np.uint8)
        assert O.migrate(s0, geom(src), sbt, want, geom(remote), dbt, 0, SH.n_layers) == O.OK
        np.testing.assert_array_equal(got, want)
        assert counts == [1] * SH.n_layers
        remote.destroy()
        q_in.put("bye")
    finally:
        proc.join(timeout=120)
        if proc.is_alive():
            proc.kill()
    assert proc.exitcode == 0
