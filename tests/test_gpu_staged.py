"""GPU parity of the staged copy-engine host path (A6 swap, kernel 4 — opt-in, selected
here for every test by the autouse fixture; wind_kv.h wind_kv_swap_out): a TMA gather /
scatter between the device pool and a device staging buffer, the copy engines over PCIe per
run of adjacent host slots, buffers pipelined on side streams.  Every result is compared with the CPU oracle over
the WHOLE host pool and device pool (untouched slots included), plus the layer flags.

Chunking (layer-major): the staging buffer holds max(32 MiB, 2 L C) bytes; a chunk is as
many whole layers of all n blocks as fit, else one layer of m = buffer // (2 C) blocks.
C1 geometry with 128 blocks (6 MiB per layer) gives 3 chunks of 5, 5 and 2 layers; a
2-layer, 288 KiB-chunk pool with 130 blocks gives 3 block chunks (56, 56, 18) per layer.
dst's layer flags move as each layer's last chunk lands: one flag kernel per layer group.
"""
import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
from windgen import migration_case, KVShape

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


@pytest.fixture(autouse=True)
def default_tuning():
    saved = {p: wk.get_tuning(p) for p in (wk.PATH_INTRA, wk.PATH_PEER, wk.PATH_HOST)}
    wk.set_tuning(wk.PATH_HOST, kernel=wk.KERNEL_STAGED)  # the staged path is opt-in
    yield
    for p, t in saved.items():
        wk.set_tuning(p, **t)


def geom(p: wk.Pool) -> O.Geom:
    d = p.desc
    return O.Geom(d.first_layer, d.n_layers, d.n_kv_heads, d.head_dim, d.block_size, d.elem_bytes,
                  d.n_blocks)


def pool(sh: KVShape, nb: int, seed: int, loc="device", first_layer=0, n_layers=None):
    p = wk.Pool(n_layers or sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes,
                nb, loc=loc, first_layer=first_layer)
    host = np.random.default_rng(seed).integers(0, 256, p.nbytes, dtype=np.uint8)
    p.tensor().copy_(torch.from_numpy(host))
    return p, host


def read(p: wk.Pool) -> np.ndarray:
    torch.cuda.synchronize()
    return p.tensor().cpu().numpy().copy()


def dtab(a) -> torch.Tensor:
    return torch.as_tensor(np.asarray(a, np.int32), device=DEV)


def htab(a) -> torch.Tensor:  # host-readable (pinned): what the staged path needs
    return torch.as_tensor(np.asarray(a, np.int32)).pin_memory()


def plan(n: int, sh: KVShape, lo: int, hi: int, host_layers: int):
    """(chunks, layer groups) of the staged path (wind_kv.cpp staged_host_op)."""
    C = sh.n_kv_heads * sh.block_size * sh.head_dim * sh.elem_bytes
    buf = max(32 << 20, 2 * host_layers * C)
    iota_n = min(1 << 16, buf // (2 * C))
    if n <= iota_n and 2 * C * n <= buf:
        lpc, m = min(hi - lo, buf // (2 * C * n)), n
    else:
        lpc, m = 1, min(iota_n, buf // (2 * C))
    groups = -(-(hi - lo) // lpc)
    return groups * -(-n // m), groups


@pytest.mark.parametrize("host_tables", ["shuffled", "runs", "sequential"])
def test_staged_round_trip_c1(host_tables):
    """C1 geometry, 128 blocks -> 3 layer-group chunks (5, 5, 2 layers): swap_out to host
    slots that are fragmented / in runs / one run, then swap_in to DIFFERENT device slots."""
    case = migration_case("C1", scale=0.5)
    sh = case.shape
    n = case.n
    nbh = n + 40
    rng = np.random.default_rng(7)
    if host_tables == "shuffled":
        hbt = rng.permutation(nbh)[:n]
    elif host_tables == "runs":  # runs of 1-9 adjacent slots, in random order
        cuts = np.sort(rng.choice(np.arange(1, nbh), 24, replace=False))
        runs = np.split(np.arange(nbh), cuts)
        hbt = np.concatenate([runs[i] for i in rng.permutation(len(runs))])[:n]
    else:
        hbt = np.arange(5, 5 + n)
    hbt = hbt.astype(np.int32)
    dev, d0 = pool(sh, case.nb_src, 1)
    host, h0 = pool(sh, nbh, 2, loc="host")
    k, groups = plan(n, sh, 0, sh.n_layers, sh.n_layers)
    assert (k, groups) == (3, 3)
    l0 = wk.launch_count()
    wk.swap_out(dev, dtab(case.src_bt), host, htab(hbt))
    torch.cuda.synchronize()
    assert wk.launch_count() - l0 == k + groups  # k gathers + one flag kernel per layer group
    want_h = h0.copy()
    assert O.swap_out(d0, geom(dev), case.src_bt, want_h, geom(host), hbt) == O.OK
    np.testing.assert_array_equal(host.tensor().numpy(), want_h)
    assert [host.layer_count(l) for l in range(sh.n_layers)] == [1] * sh.n_layers
    dev2, e0 = pool(sh, case.nb_dst, 3)
    wk.swap_in(host, htab(hbt), dev2, dtab(case.dst_bt))
    want2 = e0.copy()
    assert O.swap_in(want_h, geom(host), hbt, want2, geom(dev2), case.dst_bt) == O.OK
    got = read(dev2)
    np.testing.assert_array_equal(got, want2)
    a = d0.reshape(sh.n_layers, 2, case.nb_src, -1)[:, :, case.src_bt]
    b = got.reshape(sh.n_layers, 2, case.nb_dst, -1)[:, :, case.dst_bt]
    np.testing.assert_array_equal(a, b)  # round-trip identity (P4)
    assert [dev2.layer_count(l) for l in range(sh.n_layers)] == [1] * sh.n_layers
    assert dev2.layer_ticket() == 1 and host.layer_ticket() == 1


def test_staged_block_chunks_within_a_layer():
    """One layer of all blocks exceeds the buffer: each layer is split into block chunks
    (56, 56, 18), layer-major; swap out and back in, byte-exact, flags once per layer."""
    sh = KVShape("c3-2l", 2, 72, 128, 2)  # C = 288 KiB: 2 C n = 73 MiB per layer > 32 MiB
    n = 130
    assert plan(n, sh, 0, 2, 2) == (6, 2)
    rng = np.random.default_rng(4)
    dev, d0 = pool(sh, 140, 4)
    host, h0 = pool(sh, 135, 5, loc="host")
    sbt = rng.permutation(140)[:n].astype(np.int32)
    hbt = rng.permutation(135)[:n].astype(np.int32)
    l0 = wk.launch_count()
    wk.swap_out(dev, dtab(sbt), host, htab(hbt))
    torch.cuda.synchronize()
    assert wk.launch_count() - l0 == 6 + 2
    want = h0.copy()
    assert O.swap_out(d0, geom(dev), sbt, want, geom(host), hbt) == O.OK
    np.testing.assert_array_equal(host.tensor().numpy(), want)
    dev2, e0 = pool(sh, 131, 6)
    dbt = rng.permutation(131)[:n].astype(np.int32)
    wk.swap_in(host, htab(hbt), dev2, dtab(dbt))
    want2 = e0.copy()
    assert O.swap_in(want, geom(host), hbt, want2, geom(dev2), dbt) == O.OK
    np.testing.assert_array_equal(read(dev2), want2)
    assert [dev2.layer_count(l) for l in range(2)] == [1, 1]


def test_staged_swap_in_layer_flags_order_data():
    """Per-layer streaming on the staged path: a consumer stream waits on each layer's flag
    (wind_kv_layer_wait) and then snapshots that layer's K/V planes; every snapshot must
    already hold the swapped-in bytes (flags are published after the layer's scatter)."""
    case = migration_case("C2", scale=0.05)
    sh = case.shape  # 40 layers, C = 160 KiB
    n = case.n
    dev, d0 = pool(sh, case.nb_src, 17)
    host, _ = pool(sh, n, 18, loc="host")
    hbt = np.arange(n, dtype=np.int32)
    wk.swap_out(dev, dtab(case.src_bt), host, htab(hbt))
    dev2, e0 = pool(sh, case.nb_dst, 19)
    torch.cuda.synchronize()
    want = e0.copy()
    a = d0.reshape(sh.n_layers, 2, case.nb_src, -1)[:, :, case.src_bt]
    want.reshape(sh.n_layers, 2, case.nb_dst, -1)[:, :, case.dst_bt] = a
    plane = 2 * case.nb_dst * sh.chunk_bytes
    s, cons = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
    snaps = torch.empty(sh.n_layers, plane, dtype=torch.uint8, device=DEV)
    view = dev2.tensor()
    h_t, d_t = htab(hbt), dtab(case.dst_bt)  # borrowed until the ops complete
    for trial in range(3):
        wk.swap_in(host, h_t, dev2, d_t, stream=s)
        t = dev2.layer_ticket()
        with torch.cuda.stream(cons):
            for l in range(sh.n_layers):
                wk.layer_wait(dev2, l, t, stream=cons)
                snaps[l].copy_(view[l * plane:(l + 1) * plane])
        torch.cuda.synchronize()
        np.testing.assert_array_equal(snaps.cpu().numpy().reshape(-1), want)
        assert dev2.layer_count(0) == trial + 1


@pytest.mark.parametrize("lo,hi", [(4, 10), (6, 7), (8, 10)])
def test_staged_layer_window_and_shifted_pools(lo, hi):
    """migrate() between a device pool of global layers [4, 10) and a host pool of [0, 12)
    (PP-stage windows), layer sub-ranges, both directions; flags of every dst layer +1."""
    base = migration_case("C1", scale=0.25)
    sh = base.shape
    n = base.n
    dev, d0 = pool(sh, base.nb_src, 7, first_layer=4, n_layers=6)
    host, h0 = pool(sh, n + 3, 8, loc="host", first_layer=0, n_layers=12)
    hbt = np.random.default_rng(lo).permutation(n + 3)[:n].astype(np.int32)
    wk.migrate(dev, dtab(base.src_bt), host, htab(hbt), layer_lo=lo, layer_hi=hi)
    torch.cuda.synchronize()
    want = h0.copy()
    assert O.migrate(d0, geom(dev), base.src_bt, want, geom(host), hbt, lo, hi) == O.OK
    np.testing.assert_array_equal(host.tensor().numpy(), want)
    assert [host.layer_count(l) for l in range(12)] == [1] * 12
    dev_want = d0.copy()
    back = base.src_bt[::-1].copy()  # host -> device into other slots of the same pool
    assert O.migrate(want, geom(host), hbt, dev_want, geom(dev), back, lo, hi) == O.OK
    wk.migrate(host, htab(hbt), dev, dtab(back), layer_lo=lo, layer_hi=hi)
    np.testing.assert_array_equal(read(dev), dev_want)
    assert [dev.layer_count(l) for l in range(4, 10)] == [1] * 6


def test_staged_consecutive_ops_on_two_streams():
    """Staged ops on one host pool serialise on its staging buffers: swap_out on stream A,
    then swap_in from the same host pool on stream B with NO host-side ordering — the
    swap_in must read the bytes the swap_out wrote."""
    case = migration_case("C1", scale=0.5)
    sh = case.shape
    n = case.n
    dev, d0 = pool(sh, case.nb_src, 9)
    host, _ = pool(sh, n, 10, loc="host")
    dev2, e0 = pool(sh, case.nb_dst, 11)
    hbt = np.arange(n, dtype=np.int32)
    ta, tb = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
    s_src, s_dst, s_h = dtab(case.src_bt), dtab(case.dst_bt), htab(hbt)
    torch.cuda.synchronize()
    for _ in range(3):
        wk.swap_out(dev, s_src, host, s_h, stream=ta)
        wk.swap_in(host, s_h, dev2, s_dst, stream=tb)
    torch.cuda.synchronize()
    want = e0.copy()
    a = d0.reshape(sh.n_layers, 2, case.nb_src, -1)[:, :, case.src_bt]
    want.reshape(sh.n_layers, 2, case.nb_dst, -1)[:, :, case.dst_bt] = a
    np.testing.assert_array_equal(read(dev2), want)


def test_staged_graph_capture():
    """swap_out + swap_in captured into one CUDA graph (fork / join on the side stream) and
    replayed: byte-exact, flags bumped once per replay."""
    case = migration_case("C1", scale=0.5)
    sh = case.shape
    n = case.n
    dev, d0 = pool(sh, case.nb_src, 12)
    host, h0 = pool(sh, n, 13, loc="host")
    dev2, e0 = pool(sh, case.nb_dst, 14)
    hbt = np.random.default_rng(3).permutation(n).astype(np.int32)
    s_src, s_dst, s_h = dtab(case.src_bt), dtab(case.dst_bt), htab(hbt)
    s = torch.cuda.Stream(DEV)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g, stream=s):
        wk.swap_out(dev, s_src, host, s_h, stream=s)
        wk.swap_in(host, s_h, dev2, s_dst, stream=s)
    torch.cuda.synchronize()
    for _ in range(2):
        g.replay()
    torch.cuda.synchronize()
    want_h = h0.copy()
    assert O.swap_out(d0, geom(dev), case.src_bt, want_h, geom(host), hbt) == O.OK
    np.testing.assert_array_equal(host.tensor().numpy(), want_h)
    want2 = e0.copy()
    assert O.swap_in(want_h, geom(host), hbt, want2, geom(dev2), case.dst_bt) == O.OK
    np.testing.assert_array_equal(read(dev2), want2)
    assert host.layer_count(0) == 2 and dev2.layer_count(sh.n_layers - 1) == 2


def test_staged_errors():
    """kernel 4 forced with a device-resident host table: UNSUPPORTED; a host table entry
    out of range: BLOCK_RANGE with nothing enqueued (the table is read on the CPU)."""
    case = migration_case("C1", scale=0.25)
    sh = case.shape
    dev, _ = pool(sh, case.nb_src, 15)
    host, h0 = pool(sh, case.n, 16, loc="host")
    wk.set_tuning(wk.PATH_HOST, kernel=wk.KERNEL_STAGED)
    with pytest.raises(wk.WindKVError) as e:
        wk.swap_out(dev, dtab(case.src_bt), host, dtab(np.arange(case.n)))
    assert e.value.status == -10  # UNSUPPORTED
    bad = np.arange(case.n, dtype=np.int32)
    bad[-1] = case.n
    l0 = wk.launch_count()
    with pytest.raises(wk.WindKVError) as e:
        wk.swap_out(dev, dtab(case.src_bt), host, htab(bad))
    assert e.value.status == -4  # BLOCK_RANGE
    assert wk.launch_count() == l0 and host.layer_ticket() == 0
    torch.cuda.synchronize()
    np.testing.assert_array_equal(host.tensor().numpy(), h0)
    # kernel 4 on device -> device: UNSUPPORTED (never silently another kernel)
    other, _ = pool(sh, case.nb_src, 17)
    with pytest.raises(wk.WindKVError) as e:
        wk.migrate_ex(dev, dtab(case.src_bt), other, dtab(case.src_bt),
                      wk.tuning(kernel=wk.KERNEL_STAGED))
    assert e.value.status == -10
    # the auto choice is the SM kernel over mapped memory, whatever the host table is
    wk.set_tuning(wk.PATH_HOST, kernel=wk.KERNEL_AUTO)
    for ht in (dtab(np.arange(case.n)), htab(np.arange(case.n))):
        l0 = wk.launch_count()
        wk.swap_out(dev, dtab(case.src_bt), host, ht)
        torch.cuda.synchronize()
        assert wk.launch_count() - l0 == 1


def test_default_host_path_reads_tables_when_it_executes():
    """The default (auto) HOST path honours the borrowing contract: the tables are read when
    the op executes on the stream, not at enqueue.  The stream is held by a sleep kernel, the
    pinned host table is rewritten on the CPU after the swap_out was enqueued, and the
    result must follow the REWRITTEN table (the staged path, which reads it at enqueue,
    is opt-in for exactly this reason)."""
    wk.set_tuning(wk.PATH_HOST, kernel=wk.KERNEL_AUTO)
    case = migration_case("C1", scale=0.25)
    sh = case.shape
    n = case.n
    dev, d0 = pool(sh, case.nb_src, 23)
    host, h0 = pool(sh, n + 8, 24, loc="host")
    first = np.arange(n, dtype=np.int32)
    final = np.random.default_rng(25).permutation(n + 8)[:n].astype(np.int32)
    ht = htab(first)
    st = dtab(case.src_bt)
    s = torch.cuda.Stream(DEV)
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        torch.cuda._sleep(200_000_000)  # ~0.1 s of device time before the swap runs
    wk.swap_out(dev, st, host, ht, stream=s)
    ht.copy_(torch.from_numpy(final))   # still before execution: the op must see this
    s.synchronize()
    want = h0.copy()
    assert O.swap_out(d0, geom(dev), case.src_bt, want, geom(host), final) == O.OK
    np.testing.assert_array_equal(host.tensor().numpy(), want)


def test_no_staging_flag_uses_the_sm_path():
    """WIND_POOL_NO_STAGING: the host pool gets no device staging, so kernel 4 is refused
    (UNSUPPORTED, nothing enqueued) and the auto choice takes the SM kernel over mapped
    memory (one launch), byte-exact."""
    case = migration_case("C1", scale=0.25)
    sh = case.shape
    dev, d0 = pool(sh, case.nb_src, 20)
    host = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, case.n,
                   loc="host", staging=False)
    h0 = np.random.default_rng(21).integers(0, 256, host.nbytes, dtype=np.uint8)
    host.tensor().copy_(torch.from_numpy(h0))
    hbt = np.random.default_rng(22).permutation(case.n).astype(np.int32)
    st, ht = dtab(case.src_bt), htab(hbt)
    with pytest.raises(wk.WindKVError) as e:  # kernel 4 asked for, but no staging: refused
        wk.swap_out(dev, st, host, ht)
    assert e.value.status == -10
    wk.set_tuning(wk.PATH_HOST, kernel=wk.KERNEL_AUTO)
    l0 = wk.launch_count()
    wk.swap_out(dev, st, host, ht)
    torch.cuda.synchronize()
    assert wk.launch_count() - l0 == 1
    want = h0.copy()
    assert O.swap_out(d0, geom(dev), case.src_bt, want, geom(host), hbt) == O.OK
    np.testing.assert_array_equal(host.tensor().numpy(), want)
