"""GPU parity: every ABI entry point against the CPU oracle, byte-exact over the WHOLE
destination pool (untouched slots included), through the C ABI.

Payloads are raw bytes (fp16 / bf16 / fp8 never interpreted, R13): random bytes cover
every NaN / Inf bit pattern.  Sizes span several work units and ragged tails.
"""
import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
from windgen import migration_case, SHAPES, KVShape

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def geom(pool: wk.Pool) -> O.Geom:
    d = pool.desc
    return O.Geom(d.first_layer, d.n_layers, d.n_kv_heads, d.head_dim, d.block_size, d.elem_bytes,
                  d.n_blocks)


def make_pool(sh: KVShape, nb: int, seed: int, loc="device", first_layer=0, n_layers=None,
              debug=False):
    p = wk.Pool(n_layers or sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes,
                nb, loc=loc, first_layer=first_layer, debug=debug)
    host = np.random.default_rng(seed).integers(0, 256, p.nbytes, dtype=np.uint8)
    p.tensor().copy_(torch.from_numpy(host))
    return p, host


def read(p: wk.Pool) -> np.ndarray:
    torch.cuda.synchronize()
    return p.tensor().cpu().numpy().copy()


def tab(a) -> torch.Tensor:
    return torch.as_tensor(np.asarray(a, np.int32), device=DEV)


@pytest.fixture(autouse=True)
def default_tuning():
    saved = {p: wk.get_tuning(p) for p in (wk.PATH_INTRA, wk.PATH_PEER, wk.PATH_HOST)}
    yield
    for p, t in saved.items():
        wk.set_tuning(p, **t)


KERNELS = [(wk.KERNEL_TMA, 32768, 6), (wk.KERNEL_TMA, 8192, 4), (wk.KERNEL_TMA, 65536, 3),
           (wk.KERNEL_SIMT, 32768, 6), (wk.KERNEL_SIMT, 4096, 6), (wk.KERNEL_SIMT, 131072, 6)]


@pytest.mark.parametrize("kernel,unit,stages", KERNELS)
@pytest.mark.parametrize("variant", ["shuffled", "sequential"])
def test_migrate_c1_all_kernels(kernel, unit, stages, variant):
    """C1 (OPT-125M, C = 24 KiB): units of 4-128 KiB exercise the split-chunk path
    (parts > 1), one chunk per unit, and warp-coalesced windows (group > 1)."""
    wk.set_tuning(wk.PATH_INTRA, kernel=kernel, stage_bytes=unit, stages=stages,
                  ctas_per_sm=1 if kernel == wk.KERNEL_TMA else 4)
    case = migration_case("C1", variant=variant, scale=0.5)
    sh = case.shape
    src, s0 = make_pool(sh, case.nb_src, 1)
    dst, d0 = make_pool(sh, case.nb_dst, 2)
    for lo, hi in [(0, sh.n_layers), (3, 8), (11, 12)]:
        want = read(dst)
        assert O.migrate(s0, geom(src), case.src_bt, want, geom(dst), case.dst_bt, lo, hi) == O.OK
        wk.migrate(src, tab(case.src_bt), dst, tab(case.dst_bt), layer_lo=lo, layer_hi=hi)
        np.testing.assert_array_equal(read(dst), want)


@pytest.mark.parametrize("kernel", [wk.KERNEL_TMA, wk.KERNEL_SIMT])
@pytest.mark.parametrize("run", [1, 31, 32, 33, 65])
def test_run_coalescing_across_warp_windows(kernel, run):
    """C5 geometry (fp8, C = 16 KiB) with 64 KiB units -> 4-entry windows; runs of
    31/32/33/65 adjacent blocks straddle windows and warp boundaries."""
    wk.set_tuning(wk.PATH_INTRA, kernel=kernel, stage_bytes=65536, stages=3)
    sh = KVShape("c5-small", 3, 8, 128, 1)
    rng = np.random.default_rng(run)
    nb = 400
    starts_s = rng.permutation(nb // 80)[:4] * 80
    starts_d = rng.permutation(nb // 80)[:4] * 80
    sbt = np.concatenate([np.arange(s, s + run) for s in starts_s]).astype(np.int32)
    dbt = np.concatenate([np.arange(d, d + run) for d in starts_d]).astype(np.int32)
    sbt[len(sbt) // 2] = nb - 1  # break one run in the middle
    src, s0 = make_pool(sh, nb, 3)
    dst, d0 = make_pool(sh, nb, 4)
    want = d0.copy()
    assert O.migrate(s0, geom(src), sbt, want, geom(dst), dbt, 0, 3) == O.OK
    wk.migrate(src, tab(sbt), dst, tab(dbt))
    np.testing.assert_array_equal(read(dst), want)


@pytest.mark.parametrize("cfg", ["C2", "C3", "C4", "C5"])
def test_migrate_each_config_geometry(cfg):
    """Every BJ:configs geometry (C = 16..288 KiB, fp16 / bf16 / fp8), few layers, default
    tuning, a ragged table length."""
    full = SHAPES[cfg]
    sh = KVShape(full.name, 3, full.n_kv_heads, full.head_dim, full.elem_bytes)
    n = 37
    case = migration_case(cfg, lengths=np.array([16 * n - 5]), shape=sh)
    src, s0 = make_pool(sh, case.nb_src, 5, first_layer=10)
    dst, d0 = make_pool(sh, case.nb_dst, 6, first_layer=11, n_layers=3)
    want = d0.copy()
    assert O.migrate(s0, geom(src), case.src_bt, want, geom(dst), case.dst_bt, 11, 13) == O.OK
    wk.migrate(src, tab(case.src_bt), dst, tab(case.dst_bt), layer_lo=11, layer_hi=13)
    np.testing.assert_array_equal(read(dst), want)
    # flags: every dst layer bumped exactly once (out-of-range layer 13 at op start)
    assert [dst.layer_count(l) for l in range(11, 14)] == [1, 1, 1]
    assert dst.layer_ticket() == 1


@pytest.mark.parametrize("kernel", [wk.KERNEL_TMA, wk.KERNEL_SIMT])
def test_compact_same_pool(kernel):
    """A7: plan_compact + compact on one pool equals the oracle's snapshot semantics."""
    wk.set_tuning(wk.PATH_INTRA, kernel=kernel)
    from windgen import live_mask_after_free, lengths_longtail, blocks_for_tokens
    sh = KVShape("c5-small", 4, 8, 128, 1)
    reqb = np.minimum(blocks_for_tokens(lengths_longtail(80, 5), 16), 30)
    nb = int(reqb.sum()) + 100
    live, _ = live_mask_after_free(nb, reqb, 0.5, 9)
    sbt, dbt = wk.plan_compact(live)
    s2, d2 = O.plan_compact(live)
    np.testing.assert_array_equal(sbt, s2)
    np.testing.assert_array_equal(dbt, d2)
    pool, p0 = make_pool(sh, nb, 7)
    want = p0.copy()
    assert O.compact(want, geom(pool), sbt, dbt) == O.OK
    wk.compact(pool, tab(sbt), tab(dbt))
    np.testing.assert_array_equal(read(pool), want)


def test_identity_and_fanout_same_pool():
    sh = KVShape("t", 2, 4, 64, 2)
    pool, p0 = make_pool(sh, 50, 8)
    ident = np.arange(50, dtype=np.int32)
    wk.compact(pool, tab(ident), tab(ident))
    np.testing.assert_array_equal(read(pool), p0)
    sbt = np.array([3, 3, 3, 7], np.int32)    # fan-out (backups)
    dbt = np.array([10, 11, 12, 7], np.int32)  # (7 -> 7) identity pair
    want = p0.copy()
    assert O.compact(want, geom(pool), sbt, dbt) == O.OK
    wk.compact(pool, tab(sbt), tab(dbt))
    np.testing.assert_array_equal(read(pool), want)


@pytest.mark.parametrize("kernel", [wk.KERNEL_SIMT, wk.KERNEL_TMA])
def test_swap_round_trip(kernel):
    """A6 / P4: swap_out to a mapped host pool, swap_in to DIFFERENT device slots; both
    byte-exact vs the oracle, host pool included."""
    wk.set_tuning(wk.PATH_HOST, kernel=kernel)
    case = migration_case("C1", scale=0.5)
    sh = case.shape
    dev, d0 = make_pool(sh, case.nb_src, 9)
    host = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes,
                   case.n + 7, loc="host")
    host.tensor().zero_()
    host_bt = np.random.default_rng(1).permutation(case.n + 7)[:case.n].astype(np.int32)
    wk.swap_out(dev, tab(case.src_bt), host, tab(host_bt))
    torch.cuda.synchronize()
    want_h = np.zeros(host.nbytes, np.uint8)
    assert O.swap_out(d0, geom(dev), case.src_bt, want_h, geom(host), host_bt) == O.OK
    np.testing.assert_array_equal(host.tensor().numpy(), want_h)
    dev2, e0 = make_pool(sh, case.nb_dst, 10)
    wk.swap_in(host, tab(host_bt), dev2, tab(case.dst_bt))
    want2 = e0.copy()
    assert O.swap_in(want_h, geom(host), host_bt, want2, geom(dev2), case.dst_bt) == O.OK
    got = read(dev2)
    np.testing.assert_array_equal(got, want2)
    a = d0.reshape(sh.n_layers, 2, case.nb_src, -1)[:, :, case.src_bt]
    b = got.reshape(sh.n_layers, 2, case.nb_dst, -1)[:, :, case.dst_bt]
    np.testing.assert_array_equal(a, b)  # round-trip identity
    assert host.layer_count(0) == 1 and dev2.layer_count(sh.n_layers - 1) == 1


def test_tables_in_mapped_host_memory():
    """Block tables may live in mapped pinned host memory (wind_kv.h ownership rules)."""
    case = migration_case("C1", scale=0.25)
    sh = case.shape
    src, s0 = make_pool(sh, case.nb_src, 11)
    dst, d0 = make_pool(sh, case.nb_dst, 12)
    hs = torch.as_tensor(case.src_bt).pin_memory()
    hd = torch.as_tensor(case.dst_bt).pin_memory()
    wk.migrate(src, hs.data_ptr(), dst, hd.data_ptr(), n=case.n)
    want = d0.copy()
    assert O.migrate(s0, geom(src), case.src_bt, want, geom(dst), case.dst_bt, 0, 12) == O.OK
    np.testing.assert_array_equal(read(dst), want)


# --------------------------------------------------------------- edge cases / errors

def test_noop_cases_take_no_ticket():
    sh = KVShape("t", 2, 2, 64, 2)
    src, _ = make_pool(sh, 8, 1)
    dst, d0 = make_pool(sh, 8, 2)
    n0 = wk.launch_count()
    wk.migrate(src, tab([]), dst, tab([]), n=0)
    wk.migrate(src, tab([1]), dst, tab([2]), layer_lo=1, layer_hi=1)
    assert wk.launch_count() == n0 and dst.layer_ticket() == 0
    np.testing.assert_array_equal(read(dst), d0)
    wk.migrate(src, tab([5]), dst, tab([0]))  # one block
    assert dst.layer_ticket() == 1 and wk.launch_count() == n0 + 1


def status_of(fn, *a, **k) -> int:
    try:
        fn(*a, **k)
        return 0
    except wk.WindKVError as e:
        return e.status


def test_argument_errors_match_oracle_precedence():
    sh = KVShape("t", 4, 2, 64, 2)
    a, _ = make_pool(sh, 8, 1)
    b, b0 = make_pool(sh, 8, 2, first_layer=2)
    c = wk.Pool(4, 4, 64, 16, 2, 8)  # different H
    t1 = tab([1])
    cases = [
        ((a, t1, c, t1), dict(layer_lo=0, layer_hi=9)),   # geometry beats layer range
        ((a, t1, b, t1), dict(layer_lo=0, layer_hi=4)),   # layers 0,1 not in b
        ((a, t1, b, t1), dict(layer_lo=3, layer_hi=2)),
        ((a, t1, b, t1), dict(layer_lo=2, layer_hi=4)),   # OK
        ((a, t1, b, t1), dict(layer_lo=5, layer_hi=5)),   # empty range: no-op OK
    ]
    for args, kw in cases:
        got = status_of(wk.migrate, *args, **kw)
        want = O.check_op(geom(args[0]), geom(args[2]), 1, kw["layer_lo"], kw["layer_hi"])
        assert got == want, (kw, got, want)
    assert status_of(wk.migrate, a, t1, b, t1, n=-1) == -1
    # a pool on a device that does not exist -> INVALID_ARG at creation
    with pytest.raises(wk.WindKVError) as e:
        wk.Pool(4, 2, 64, 16, 2, 8, device=torch.cuda.device_count() + 3)
    assert e.value.status == -1
    torch.cuda.synchronize()


def test_invalid_arg_precedes_geometry_and_layer_range():
    """S§8(b) "Errors": every INVALID_ARG condition (NULL table, n < 0, repeated batch
    destination, stream of another device) wins over GEOMETRY / LAYER_RANGE, with nothing
    enqueued."""
    sh = KVShape("t", 4, 2, 64, 2)
    a, _ = make_pool(sh, 8, 1)
    b, _ = make_pool(sh, 8, 2, first_layer=2)
    c = wk.Pool(4, 4, 64, 16, 2, 8)  # different H: GEOMETRY against a
    t1 = tab([1])
    n0 = wk.launch_count()
    # NULL table + geometry mismatch, NULL table + bad layer range
    assert status_of(wk.migrate, a, None, c, t1, n=1, layer_lo=0, layer_hi=4) == -1
    assert status_of(wk.migrate, a, t1, b, None, n=1, layer_lo=0, layer_hi=9) == -1
    assert status_of(wk.migrate, a, None, b, t1, n=1, layer_lo=3, layer_hi=1) == -1
    # n < 0 + geometry mismatch
    assert status_of(wk.migrate, a, t1, c, t1, n=-1) == -1
    # head range: n_heads < 1 beats a head range that leaves the pool
    assert status_of(wk.migrate_heads, a, t1, c, t1, 0, 7, 0) == -1
    # batch: a repeated destination beats another item's geometry mismatch
    assert status_of(wk.migrate_batch, a, [(b, t1, t1), (c, t1, t1), (b, t1, t1)], 2, 4) == -1
    # the same calls without the INVALID_ARG condition report the next class
    assert status_of(wk.migrate, a, t1, c, t1, n=1, layer_lo=0, layer_hi=4) == -2
    assert status_of(wk.migrate, a, t1, b, t1, n=1, layer_lo=0, layer_hi=9) == -3
    assert status_of(wk.migrate_batch, a, [(b, t1, t1), (c, t1, t1)], 2, 4) == -2
    assert wk.launch_count() == n0
    assert a.layer_ticket() == b.layer_ticket() == c.layer_ticket() == 0
    torch.cuda.synchronize()


def test_argument_precedence_random_vs_oracle():
    """300 random argument combinations (NULL tables, n < 0 / 0 / > 0, same-geometry /
    other-H / same pool, layer windows in and out of range, inverted and empty ranges): the
    library's status equals the oracle's (or_migrate, which states S§8(b)'s precedence)."""
    import ctypes as ct
    sh = KVShape("t", 4, 2, 64, 2)
    a, a0 = make_pool(sh, 6, 1)
    b, b0 = make_pool(sh, 6, 2, first_layer=2)
    c = wk.Pool(4, 4, 64, 16, 2, 6)  # different H
    c0 = np.zeros(c.nbytes, np.uint8)
    host = {id(a): a0, id(b): b0, id(c): c0}
    sbt_d, dbt_d = tab([0, 1]), tab([2, 3])
    sbt_h, dbt_h = np.array([0, 1], np.int32), np.array([2, 3], np.int32)
    lib = O._lib()
    rng = np.random.default_rng(77)
    seen = set()
    for _ in range(300):
        dst = [a, b, c][int(rng.integers(0, 3))]
        n = int(rng.choice([-1, 0, 1, 2]))
        null_s, null_d = bool(rng.random() < 0.25), bool(rng.random() < 0.25)
        lo = int(rng.integers(-1, 8))
        hi = int(rng.integers(-1, 8))
        got = status_of(wk.migrate, a, None if null_s else sbt_d.data_ptr(), dst,
                        None if null_d else dbt_d.data_ptr(), n=n, layer_lo=lo, layer_hi=hi)
        src_h = host[id(a)]
        dst_h = src_h if dst is a else host[id(dst)].copy()
        want = lib.or_migrate(O._p(src_h), ct.byref(geom(a).c()),
                              None if null_s else O._p(sbt_h), O._p(dst_h), ct.byref(geom(dst).c()),
                              None if null_d else O._p(dbt_h), n, lo, hi)
        assert got == want, dict(dst="abc"[[a, b, c].index(dst)], n=n, null=(null_s, null_d), lo=lo, hi=hi,
                                 got=got, want=want)
        seen.add(got)
    assert {0, -1, -2, -3} <= seen  # every precedence class was exercised
    torch.cuda.synchronize()


def test_wrong_device_stream_precedes_geometry():
    """A stream of another device is INVALID_ARG even when the pools also mismatch (needs
    two GPUs to build such a stream)."""
    if torch.cuda.device_count() < 2:
        pytest.skip("needs 2 GPUs for a stream of another device")
    sh = KVShape("t", 4, 2, 64, 2)
    a, _ = make_pool(sh, 8, 1)
    c = wk.Pool(4, 4, 64, 16, 2, 8)
    t1 = tab([1])
    other = torch.cuda.Stream(device=1)
    assert status_of(wk.migrate, a, t1, c, t1, n=1, stream=other) == -1
    assert status_of(wk.migrate, a, t1, c, t1, n=1) == -2
    assert status_of(wk.migrate, a, t1, a, tab([2]), n=1, layer_lo=0, layer_hi=9, stream=other) == -1


def test_validate_matches_oracle_random_tables():
    sh = KVShape("t", 2, 2, 64, 2)
    a, _ = make_pool(sh, 6, 1)
    b, _ = make_pool(sh, 5, 2)
    rng = np.random.default_rng(0)
    for trial in range(400):
        same = trial % 2 == 0
        d = a if same else b
        n = int(rng.integers(0, 5))
        sbt = rng.integers(-1, 7, n)
        dbt = rng.integers(-1, d.desc.n_blocks + 1, n)
        got = wk.validate(a, sbt, d, dbt, 0, 2)
        want = O.validate(geom(a), sbt, geom(d), dbt, same)
        assert got == want, (sbt, dbt, same)


@pytest.mark.parametrize("bad,code", [("range", -4), ("dup", -5), ("alias", -6)])
def test_debug_pool_device_check(bad, code):
    sh = KVShape("t", 2, 2, 64, 2)
    pool, _ = make_pool(sh, 16, 3, debug=True)
    sbt, dbt = {"range": ([1, 2], [3, 99]), "dup": ([1, 2], [5, 5]),
                "alias": ([1, 2], [2, 9])}[bad]
    wk.compact(pool, tab(sbt), tab(dbt))
    with pytest.raises(wk.WindKVError) as e:
        wk.check_device_error(pool)
    assert e.value.status == -11 and e.value.status != code  # DEVICE_CHECK
    assert {"range": "BLOCK_RANGE", "dup": "DUP_DST", "alias": "ALIAS"}[bad] in str(e.value)
    wk.compact(pool, tab([1, 2]), tab([3, 4]))
    wk.check_device_error(pool)  # clean op -> OK


def test_batch_migrate_matches_sequential_oracle():
    """A8: one launch pushing to several destination pools (all-to-all sender side)."""
    sh = KVShape("t", 3, 8, 128, 2)
    src, s0 = make_pool(sh, 300, 1)
    dsts = [make_pool(sh, 120 + 10 * k, 20 + k) for k in range(5)]
    rng = np.random.default_rng(2)
    perm = rng.permutation(300).astype(np.int32)
    items, pos = [], 0
    for k, (d, d0) in enumerate(dsts):
        m = [40, 0, 77, 3, 100][k]
        sb = perm[pos:pos + m]
        pos += m
        db = rng.permutation(d.desc.n_blocks)[:m].astype(np.int32)
        items.append((d, tab(sb), tab(db), sb, db, d0))
    wk.migrate_batch(src, [(d, ts, td) for d, ts, td, *_ in items], 0, 3)
    for d, _, _, sb, db, d0 in items:
        want = d0.copy()
        assert O.migrate(s0, geom(src), sb, want, geom(d), db, 0, 3) == O.OK
        np.testing.assert_array_equal(read(d), want)
        assert d.layer_ticket() == 1 and [d.layer_count(l) for l in range(3)] == [1, 1, 1]


@pytest.mark.parametrize("variant", ["shuffled", "sequential"])
def test_copy_engine_path_matches_oracle(variant):
    """kernel = 3 (DMA engines, zero SMs): same result as the oracle; host-readable tables
    required; flags published once per op."""
    wk.set_tuning(wk.PATH_INTRA, kernel=wk.KERNEL_COPY_ENGINE)
    case = migration_case("C1", variant=variant, scale=0.5)
    sh = case.shape
    src, s0 = make_pool(sh, case.nb_src, 21)
    dst, d0 = make_pool(sh, case.nb_dst, 22)
    want = d0.copy()
    assert O.migrate(s0, geom(src), case.src_bt, want, geom(dst), case.dst_bt, 2, 10) == O.OK
    hs = torch.as_tensor(case.src_bt).pin_memory()
    hd = torch.as_tensor(case.dst_bt).pin_memory()
    n0 = wk.launch_count()
    wk.migrate(src, hs.data_ptr(), dst, hd.data_ptr(), n=case.n, layer_lo=2, layer_hi=10)
    np.testing.assert_array_equal(read(dst), want)
    assert wk.launch_count() - n0 == 1  # the flag kernel only
    assert [dst.layer_count(l) for l in range(sh.n_layers)] == [1] * sh.n_layers
    with pytest.raises(wk.WindKVError) as e:  # device tables: not readable by the host
        wk.migrate(src, tab(case.src_bt), dst, tab(case.dst_bt))
    assert e.value.status == -10
