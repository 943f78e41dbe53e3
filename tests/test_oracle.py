"""Pins for the CPU oracle, CPU only.

Each test pins the oracle to something other than itself: an element-wise brute force
(tests/brute.py), numpy advanced indexing, invariants, closed forms and the values the
paper prints (tests/golden/).
"""
import itertools
import json
import os

import numpy as np
import pytest

import oracle as O
import brute
from windgen import content_bytes, migration_case, SHAPES

HERE = os.path.dirname(os.path.abspath(__file__))


def rand_pool(g: O.Geom, seed: int) -> np.ndarray:
    return np.random.default_rng(seed).integers(0, 256, g.pool_bytes, dtype=np.uint8)


TINY = dict(n_kv_heads=2, head_dim=4, block_size=2, elem_bytes=2)  # C = 32 B


# ----------------------------------------------------------------- P3 brute force

@pytest.mark.parametrize("same_pool", [False, True])
def test_exhaustive_tiny_tables(same_pool):
    """P3: every table pair with n <= 2 over 3-slot pools (plus every n = 3 table with
    distinct-pool sources fixed), 3 layer ranges, against the element-wise brute force,
    status code AND bytes."""
    gs = O.Geom(first_layer=1, n_layers=2, n_blocks=3, **TINY)
    gd = gs if same_pool else O.Geom(first_layer=0, n_layers=3, n_blocks=3, **TINY)
    src0 = rand_pool(gs, 1)
    dst0 = src0 if same_pool else rand_pool(gd, 2)
    ranges = [(1, 3), (2, 3), (1, 1)]
    n_cases = 0
    for n in range(0, 3):
        for sbt in itertools.product(range(-1, 4), repeat=n):
            for dbt in itertools.product(range(3), repeat=n):
                for lo, hi in ranges:
                    src = src0.copy()
                    dst = src if same_pool else dst0.copy()
                    st_b, want = brute.brute_migrate(src, gs, sbt, dst, gd, dbt, lo, hi,
                                                     same_pool)
                    st = O.migrate(src, gs, sbt, dst, gd, dbt, lo, hi)
                    assert st == st_b, (sbt, dbt, lo, hi)
                    np.testing.assert_array_equal(dst, want)
                    n_cases += 1
    assert n_cases > 700


def test_random_n3_brute():
    rng = np.random.default_rng(7)
    gs = O.Geom(first_layer=0, n_layers=2, n_blocks=5, **TINY)
    gd = O.Geom(first_layer=0, n_layers=2, n_blocks=4, **TINY)
    for trial in range(300):
        same = trial % 2 == 1
        g2 = gs if same else gd
        sbt = rng.integers(0, gs.n_blocks, 3).tolist()
        dbt = rng.integers(0, g2.n_blocks, 3).tolist()
        lo = int(rng.integers(0, 2))
        hi = int(rng.integers(lo, 3))
        src = rand_pool(gs, trial)
        dst = src if same else rand_pool(gd, trial + 1000)
        st_b, want = brute.brute_migrate(src, gs, sbt, dst, g2, dbt, lo, hi, same)
        st = O.migrate(src, gs, sbt, dst, g2, dbt, lo, hi)
        assert st == st_b
        np.testing.assert_array_equal(dst, want)


# ------------------------------------------------------ P1 numpy advanced indexing

@pytest.mark.parametrize("variant", ["shuffled", "sequential"])
def test_numpy_formula_c1(variant):
    """P1: D.reshape(L,2,NB,C)[lo-l0:hi-l0, :, dbt] = S.reshape(L,2,NB,C)[..., sbt]."""
    case = migration_case("C1", variant=variant, scale=0.25)
    sh = case.shape
    gs = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes,
                case.nb_src)
    gd = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes,
                case.nb_dst)
    src = rand_pool(gs, 11)
    dst = rand_pool(gd, 12)
    for lo, hi in [(0, sh.n_layers), (3, 7), (5, 5)]:
        d = dst.copy()
        assert O.migrate(src, gs, case.src_bt, d, gd, case.dst_bt, lo, hi) == O.OK
        want = dst.copy().reshape(gd.n_layers, 2, gd.n_blocks, -1)
        S = src.reshape(gs.n_layers, 2, gs.n_blocks, -1)
        want[lo:hi, :, case.dst_bt] = S[lo:hi, :, case.src_bt]
        np.testing.assert_array_equal(d, want.reshape(-1))


def test_numpy_formula_same_pool_snapshot():
    """Same pool: numpy materialises the right-hand side first = snapshot semantics."""
    g = O.Geom(2, 3, 2, 8, 4, 1, 12)
    pool = rand_pool(g, 5)
    sbt = np.array([3, 7, 0, 0], np.int32)   # duplicate source = fan-out (R5)
    dbt = np.array([3, 1, 9, 10], np.int32)  # (3 -> 3) is an identity pair (R4)
    want = pool.copy().reshape(3, 2, 12, -1)
    want[0:3, :, dbt] = want[0:3, :, sbt].copy()
    assert O.migrate(pool, g, sbt, pool, g, dbt, 2, 5) == O.OK
    np.testing.assert_array_equal(pool, want.reshape(-1))


def test_first_layer_shift():
    """Pools covering different layer ranges (PP stages): global layer l lives at local
    index l - first_layer on each side."""
    gs = O.Geom(4, 4, 2, 8, 2, 2, 6)   # layers 4..7
    gd = O.Geom(6, 4, 2, 8, 2, 2, 5)   # layers 6..9
    src, dst = rand_pool(gs, 1), rand_pool(gd, 2)
    sbt, dbt = [5, 0, 2], [4, 3, 0]
    want = dst.copy().reshape(4, 2, 5, -1)
    want[0:2, :, dbt] = src.reshape(4, 2, 6, -1)[2:4, :, sbt]
    assert O.migrate(src, gs, sbt, dst, gd, dbt, 6, 8) == O.OK
    np.testing.assert_array_equal(dst, want.reshape(-1))
    assert O.migrate(src, gs, sbt, dst, gd, dbt, 5, 8) == O.LAYER_RANGE
    assert O.migrate(src, gs, sbt, dst, gd, dbt, 6, 9) == O.LAYER_RANGE


# ---------------------------------------------------------------- P4 invariants

def test_round_trip_swap():
    """P4: swap_out then swap_in into DIFFERENT device slots gives identical chunks."""
    g = O.Geom(0, 3, 2, 16, 4, 2, 10)
    gh = O.Geom(0, 3, 2, 16, 4, 2, 7)
    dev = rand_pool(g, 3)
    host = np.zeros(gh.pool_bytes, np.uint8)
    out_bt, host_bt, back_bt = [9, 2, 4, 5], [6, 0, 1, 3], [0, 1, 7, 8]
    assert O.swap_out(dev, g, out_bt, host, gh, host_bt) == O.OK
    dev2 = rand_pool(g, 4)
    assert O.swap_in(host, gh, host_bt, dev2, g, back_bt) == O.OK
    a = dev.reshape(3, 2, 10, -1)
    b = dev2.reshape(3, 2, 10, -1)
    np.testing.assert_array_equal(a[:, :, out_bt], b[:, :, back_bt])


def test_identity_noop():
    g = O.Geom(0, 4, 2, 8, 4, 2, 9)
    pool = rand_pool(g, 9)
    before = pool.copy()
    ident = np.arange(9, dtype=np.int32)
    assert O.migrate(pool, g, ident, pool, g, ident, 0, 4) == O.OK
    np.testing.assert_array_equal(pool, before)
    assert O.compact(pool, g, ident, ident) == O.OK
    np.testing.assert_array_equal(pool, before)


def test_write_once_and_conservation():
    """P4: with every source chunk distinct (content pattern), each touched destination
    chunk holds exactly one source chunk, untouched chunks keep their bytes, and the
    multiset of touched chunks equals the multiset of source chunks."""
    case = migration_case("C1", scale=0.25)
    sh = case.shape
    gs = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, case.nb_src)
    gd = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, case.nb_dst)
    src = content_bytes(1, 1, 0, gs.pool_bytes)
    dst = content_bytes(1, 2, 0, gd.pool_bytes)
    before = dst.copy()
    assert O.migrate(src, gs, case.src_bt, dst, gd, case.dst_bt, 0, sh.n_layers) == O.OK
    C = gs.chunk_bytes
    D = dst.reshape(-1, C)
    B = before.reshape(-1, C)
    S = src.reshape(-1, C)
    src_chunks = {S[i].tobytes(): i for i in range(S.shape[0])}
    touched = np.zeros(D.shape[0], bool)
    for l in range(sh.n_layers):
        for kv in range(2):
            for b in case.dst_bt:
                touched[(l * 2 + kv) * gd.n_blocks + b] = True
    assert touched.sum() == 2 * sh.n_layers * case.n
    hits = [src_chunks.get(D[c].tobytes(), -1) for c in np.flatnonzero(touched)]
    assert min(hits) >= 0 and len(set(hits)) == len(hits)
    np.testing.assert_array_equal(D[~touched], B[~touched])


def test_expected_origin_matches_migrate():
    case = migration_case("C1", scale=0.25)
    sh = case.shape
    gs = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, case.nb_src)
    gd = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, case.nb_dst)
    src = content_bytes(5, 1, 0, gs.pool_bytes)
    dst = content_bytes(5, 2, 0, gd.pool_bytes)
    for lo, hi in [(0, 12), (2, 9)]:
        d = dst.copy()
        assert O.migrate(src, gs, case.src_bt, d, gd, case.dst_bt, lo, hi) == O.OK
        fs, off = O.expected_origin(gs, case.src_bt, gd, case.dst_bt, lo, hi)
        C = gs.chunk_bytes
        for c in range(0, fs.size, 7):
            want = content_bytes(5, 1 if fs[c] else 2, int(off[c]), C)
            np.testing.assert_array_equal(d[c * C:(c + 1) * C], want)


def test_migrate_mt_equals_migrate():
    case = migration_case("C1", scale=0.5)
    sh = case.shape
    gs = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, case.nb_src)
    gd = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, case.nb_dst)
    src = rand_pool(gs, 1)
    d1, d2 = rand_pool(gd, 2), rand_pool(gd, 2)
    assert O.migrate(src, gs, case.src_bt, d1, gd, case.dst_bt, 1, 11) == O.OK
    assert O.migrate_mt(src, gs, case.src_bt, d2, gd, case.dst_bt, 1, 11, 3) == O.OK
    np.testing.assert_array_equal(d1, d2)


# -------------------------------------------------------------- error precedence

def test_error_precedence():
    gs = O.Geom(0, 2, 2, 8, 2, 2, 4)
    gd = O.Geom(0, 2, 2, 8, 2, 2, 4)
    gbad = O.Geom(0, 2, 4, 8, 2, 2, 4)
    src, dst = rand_pool(gs, 0), rand_pool(gd, 1)
    # geometry beats layer range and block range
    assert O.check_op(gs, gbad, 1, 0, 9) == O.GEOMETRY
    assert O.check_op(gs, gd, -1, 0, 1) == O.INVALID_ARG
    assert O.check_op(gs, gd, 1, 1, 0) == O.LAYER_RANGE
    assert O.check_op(gs, gd, 1, 0, 3) == O.LAYER_RANGE
    assert O.check_op(gs, gd, 1, 5, 5) == O.OK  # empty range is a no-op (R19)
    # block range beats duplicate destination beats alias
    assert O.validate(gs, [0, 9], gd, [1, 1], False) == O.BLOCK_RANGE
    assert O.validate(gs, [0, 1], gd, [2, 2], False) == O.DUP_DST
    assert O.validate(gs, [0, 1], gs, [1, 2], True) == O.ALIAS   # chain 0->1, 1->2
    assert O.validate(gs, [0, 1], gs, [1, 0], True) == O.ALIAS   # cycle
    assert O.validate(gs, [0, 1], gd, [1, 2], False) == O.OK     # distinct pools
    assert O.validate(gs, [2, 2], gd, [0, 1], False) == O.OK     # fan-out (R5)
    assert O.validate(gs, [1, 3], gs, [1, 0], True) == O.OK      # identity pair (R4)
    before = dst.copy()
    assert O.migrate(src, gs, [0, 1], dst, gd, [2, 2], 0, 2) == O.DUP_DST
    np.testing.assert_array_equal(dst, before)  # nothing written on error
    assert O.geom_check(O.Geom(0, 1, 1, 3, 1, 1, 1)) == O.UNSUPPORTED  # C = 3, not %16
    assert O.geom_check(O.Geom(0, 1, 1, 16, 1, 3, 1)) == O.UNSUPPORTED  # e_b = 3
    assert O.geom_check(O.Geom(0, 0, 1, 16, 1, 1, 1)) == O.INVALID_ARG


def test_null_tables_are_invalid_arg_before_geometry_and_layers():
    """S§8(b) "Errors": INVALID_ARG (every null handle) precedes GEOMETRY and LAYER_RANGE, so a
    NULL table of a non-empty op is INVALID_ARG even when the pools also mismatch."""
    import ctypes as ct
    gs = O.Geom(0, 2, 2, 8, 2, 2, 4)
    gbad = O.Geom(0, 2, 4, 8, 2, 2, 4)
    src, dst = rand_pool(gs, 0), rand_pool(gbad, 1)
    lib = O._lib()
    for gd, lo, hi in ((gbad, 0, 2), (gs, 0, 9), (gbad, 3, 1)):
        d = dst if gd is gbad else rand_pool(gs, 2)
        rc = lib.or_migrate(O._p(src), ct.byref(gs.c()), None, O._p(d), ct.byref(gd.c()),
                            O._p(np.zeros(1, np.int32)), 1, lo, hi)
        assert rc == O.INVALID_ARG, (lo, hi, rc)
    # n == 0 needs no tables: the geometry error stands
    rc = lib.or_migrate(O._p(src), ct.byref(gs.c()), None, O._p(dst), ct.byref(gbad.c()), None, 0, 0, 2)
    assert rc == O.GEOMETRY


# ---------------------------------------------------------- P5 closed forms / golden

def test_golden_p120_opt13b_bytes():
    """P:120 §2.2: one 2048-token OPT-13B request carries 'approximately 1.5 GB' of KV.
    The oracle's pool geometry gives 2 * L * C per block; 128 blocks of 16 tokens."""
    gold = json.load(open(os.path.join(HERE, "golden", "p120_opt13b_kv_bytes.json")))
    sh = SHAPES["C2"]
    g = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, 128)
    assert g.pool_bytes == gold["kv_bytes_2048_tokens"]
    assert g.pool_bytes / 2**30 == gold["gib"]
    assert abs(g.pool_bytes / 1e9 - gold["paper_gb_approx"]) < 0.2
    # the paper's "~65 ms" over PCIe Gen4 x16 implies ~25.8 GB/s effective (R17)
    assert abs(g.pool_bytes / gold["paper_ms"] * 1e3 / 1e9 - gold["implied_gbs"]) < 0.1


def test_golden_p162_decode_kv_read():
    """P:162 / Table 1: decode KV IO per layer = 4 * SUM(L) * H bytes (fp16, H = hidden
    size).  For OPT-13B (H = 5120) the oracle's per-layer chunk bytes per token must be
    4H: one layer's K+V chunks of a block, divided by the block's 16 tokens."""
    gold = json.load(open(os.path.join(HERE, "golden", "p162_decode_io.json")))
    for name, hidden in gold["hidden"].items():
        sh = {"OPT-13B": SHAPES["C2"], "OPT-66B": SHAPES["C3"], "OPT-125M": SHAPES["C1"]}[name]
        g = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, 1)
        assert sh.n_kv_heads * sh.head_dim == hidden
        per_token_layer = 2 * g.chunk_bytes // 16
        assert per_token_layer == 4 * hidden
        sum_l = gold["example_sum_L"]
        assert sum_l * per_token_layer == gold["expected_bytes"][name]


def test_payload_closed_form():
    """P5: payload(n, lo, hi) = 2 (hi - lo) n C, and per-element offsets compose."""
    g = O.Geom(3, 5, 3, 8, 4, 2, 7)
    C = g.chunk_bytes
    assert C == 3 * 4 * 8 * 2
    assert g.pool_bytes == 5 * 2 * 7 * C
    # element offsets are a bijection onto [0, pool_bytes) in steps of e_b
    offs = sorted(O.elem_offset(g, l, kv, b, h, t, j)
                  for l in range(3, 8) for kv in range(2) for b in range(7)
                  for h in range(3) for t in range(4) for j in range(8))
    assert offs == list(range(0, g.pool_bytes, 2))


# ---------------------------------------------------------------- P6 compaction plan

def test_plan_compact_exhaustive():
    """P6: for every live mask over 10 slots: post-state live set = [0, n_live); the move
    count equals the number of live slots >= n_live (a lower bound for any plan); the
    plan passes the same-pool preconditions (no alias)."""
    for mask in range(1 << 10):
        live = np.array([(mask >> b) & 1 for b in range(10)], np.uint8)
        src, dst = O.plan_compact(live)
        n_live = int(live.sum())
        assert len(src) == int(live[n_live:].sum())
        post = live.copy()
        post[src] = 0
        post[dst] = 1
        assert post[:n_live].all() and not post[n_live:].any()
        g = O.Geom(0, 1, 1, 16, 1, 1, 10)
        assert O.validate(g, src, g, dst, True) == O.OK


def test_compact_preserves_requests():
    """P6: every request reads identical logical KV before and after compaction, with
    its block table remapped through the plan's pairs."""
    from windgen import live_mask_after_free, lengths_longtail, blocks_for_tokens
    g = O.Geom(0, 2, 2, 16, 16, 1, 1500)
    reqb = blocks_for_tokens(lengths_longtail(60, 5), 16)
    reqb = np.minimum(reqb, 20)
    live, tables = live_mask_after_free(1500, reqb, 0.5, 9)
    pool = rand_pool(g, 3)
    before = pool.reshape(2, 2, 1500, -1).copy()
    src, dst = O.plan_compact(live)
    assert O.compact(pool, g, src, dst) == O.OK
    remap = dict(zip(src.tolist(), dst.tolist()))
    after = pool.reshape(2, 2, 1500, -1)
    n_live = int(live.sum())
    for t in tables:
        t2 = np.array([remap.get(int(b), int(b)) for b in t])
        assert (t2 < n_live).all()
        np.testing.assert_array_equal(after[:, :, t2], before[:, :, t])


# ---------------------------------------------------------------- P7 rebalance plan

def test_plan_rebalance_invariants():
    """P7 invariants (the choice is pinned separately, test_o7_rebalance_worked_examples): block conservation; at stop,
    either max load <= target or no request on the most-loaded GPU fits on the least
    loaded one under target; moves only go from above-target to at-most-target GPUs."""
    from windgen import skewed_placement, lengths_longtail, blocks_for_tokens
    for G in (2, 3, 8):
        for seed in range(5):
            R = 200
            gpu = skewed_placement(R, G, seed)
            blocks = blocks_for_tokens(lengths_longtail(R, seed), 16).astype(np.int32)
            out, moves = O.plan_rebalance(G, gpu, blocks)
            load0 = np.bincount(gpu, weights=blocks, minlength=G)
            load = np.bincount(out, weights=blocks, minlength=G)
            assert load.sum() == load0.sum()
            target = -(-int(blocks.sum()) // G)
            assert (load <= np.maximum(load0, target)).all()
            assert load.max() <= load0.max()
            src, dst = int(np.argmax(load)), int(np.argmin(load))
            if load[src] > target:
                fits = [b for r, b in enumerate(blocks) if out[r] == src and b > 0
                        and load[dst] + b <= target]
                assert not fits
            assert moves == int((out != gpu).sum())


# ------------------------------------------------------ O8 stall-free staging (NEXT-1)

def closed_form_stall_free(T0, bs, theta, appends):
    """Independent closed form of P:231's protocol (reading R6): with tok_k the tokens when
    stage k starts (prefix sums of the appends), stage k sends [floor(tok_{k-1}/bs),
    floor(tok_k/bs)); the pause comes after the first stage k with
    ceil(tok_{k+1}/bs) - floor(tok_k/bs) <= theta (or the last allowed stage)."""
    tok = T0 + np.concatenate([[0], np.cumsum(appends)])
    m = len(appends)
    fl = tok // bs
    ce = -(-tok // bs)
    stages = [(0, int(fl[0]))]
    for k in range(m):
        if ce[k + 1] - fl[k] <= theta or k + 1 == m:
            stages.append((int(fl[k]), int(ce[k + 1])))
            return stages, int(tok[k + 1])
        stages.append((int(fl[k]), int(fl[k + 1])))
    raise AssertionError


def test_stall_free_plan_matches_closed_form():
    rng = np.random.default_rng(0)
    for trial in range(3000):
        bs = int(rng.choice([1, 2, 16]))
        T0 = int(rng.integers(0, 300))
        theta = int(rng.integers(0, 6))
        m = int(rng.integers(1, 12))
        appends = rng.integers(0, 40, m)
        got = O.stall_free_plan(T0, bs, theta, appends)
        assert got == closed_form_stall_free(T0, bs, theta, appends), (T0, bs, theta, appends)


def test_stall_free_plan_invariants():
    """P9: every block of the request at the pause is sent exactly once, in order (so the
    bytes sent are ceil(final/bs) * 2 * L * C); stages before the pause carry only full
    blocks; the pause leaves at most theta blocks (unless max stages forced it)."""
    rng = np.random.default_rng(1)
    for trial in range(2000):
        bs, T0, theta = 16, int(rng.integers(0, 5000)), int(rng.integers(1, 8))
        appends = rng.integers(0, 64, 20)
        stages, final = O.stall_free_plan(T0, bs, theta, appends)
        cover = [b for s, e in stages for b in range(s, e)]
        assert cover == list(range(-(-final // bs)))
        tok = T0
        for k, (s, e) in enumerate(stages[:-1]):
            assert e <= tok // bs  # only blocks full when the stage starts
            tok += int(appends[k])
        s, e = stages[-1]
        if len(stages) - 1 < len(appends):
            assert e - s <= theta
    # theta larger than any request: one bulk stage, then the pause sends the tail
    assert O.stall_free_plan(100, 16, 10**6, [5, 5]) == ([(0, 6), (6, 7)], 105)


# ------------------------------------------------------------ NEXT-3 head-range migrate

def test_migrate_heads_brute_force():
    """Element-wise: D[l, kv, dbt[i], dh0 + h] = S[l, kv, sbt[i], sh0 + h] via 7-D numpy
    indexing, all other bytes unchanged; random geometries, offsets and tables."""
    rng = np.random.default_rng(3)
    for trial in range(200):
        Hs, Hd = int(rng.integers(1, 5)), int(rng.integers(1, 5))
        nh = int(rng.integers(1, min(Hs, Hd) + 1))
        sh0, dh0 = int(rng.integers(0, Hs - nh + 1)), int(rng.integers(0, Hd - nh + 1))
        gs = O.Geom(0, 2, Hs, 8, 2, 1, 5)
        gd = O.Geom(0, 3, Hd, 8, 2, 1, 4)
        n = int(rng.integers(0, 4))
        sbt = rng.integers(0, 5, n).astype(np.int32)
        dbt = rng.permutation(4)[:n].astype(np.int32)
        lo, hi = 0, int(rng.integers(0, 3))
        src, dst = rand_pool(gs, trial), rand_pool(gd, trial + 99)
        want = dst.copy()
        W = brute.as7d(want, gd)
        S = brute.as7d(src, gs)
        for i in range(n):
            for l in range(lo, hi):
                for kv in range(2):
                    for h in range(nh):
                        W[l, kv, dbt[i], dh0 + h] = S[l, kv, sbt[i], sh0 + h]
        assert O.migrate_heads(src, gs, sbt, dst, gd, dbt, lo, hi, sh0, dh0, nh) == O.OK
        np.testing.assert_array_equal(dst, want)


def test_tp_reshard_equals_full_migrate():
    """[TP-2 -> TP-1] (Fig. 3): two prefill ranks, each holding half the heads,
    push their halves into one decode pool; the result equals migrating the unsharded
    pool directly, and migrate_heads over all heads equals migrate."""
    H = 8
    full = O.Geom(0, 3, H, 16, 16, 2, 20)
    half = O.Geom(0, 3, H // 2, 16, 16, 2, 20)
    src = rand_pool(full, 1)
    S = src.reshape(3, 2, 20, H, -1)
    shards = [np.ascontiguousarray(S[:, :, :, r * H // 2:(r + 1) * H // 2]).reshape(-1) for r in range(2)]
    sbt, dbt = np.array([3, 7, 19, 0], np.int32), np.array([5, 6, 1, 2], np.int32)
    want = rand_pool(full, 2)
    got = want.copy()
    assert O.migrate(src, full, sbt, want, full, dbt, 0, 3) == O.OK
    for r in range(2):
        assert O.migrate_heads(shards[r], half, sbt, got, full, dbt, 0, 3, 0, r * H // 2, H // 2) == O.OK
    np.testing.assert_array_equal(got, want)
    got2 = rand_pool(full, 2)
    assert O.migrate_heads(src, full, sbt, got2, full, dbt, 0, 3, 0, 0, H) == O.OK
    np.testing.assert_array_equal(got2, want)


def test_migrate_heads_errors():
    gs, gd = O.Geom(0, 2, 4, 8, 2, 1, 5), O.Geom(0, 2, 2, 8, 2, 1, 5)
    assert O.check_op_heads(gs, gd, 1, 0, 2, 0, 0, 2) == O.OK
    assert O.check_op_heads(gs, gd, 1, 0, 2, 0, 1, 2) == O.GEOMETRY   # leaves dst heads
    assert O.check_op_heads(gs, gd, 1, 0, 2, 3, 0, 2) == O.GEOMETRY   # leaves src heads
    assert O.check_op_heads(gs, gd, 1, 0, 2, 0, 0, 0) == O.INVALID_ARG
    assert O.check_op_heads(gs, O.Geom(0, 2, 2, 16, 2, 1, 5), 1, 0, 2, 0, 0, 1) == O.GEOMETRY
    assert O.check_op_heads(gs, gd, 1, 0, 3, 0, 0, 1) == O.LAYER_RANGE


def test_o6_pairing_worked_example():
    """O6 pairs holes[k] <- movers[k] (both ascending).  Invariant checks alone accept any
    valid pairing (e.g. holes ascending <- movers descending); these hand-worked examples
    (tests/golden/o6_compaction_worked_example.json, S§8(c) O6) pin the pairing itself."""
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "o6_compaction_worked_example.json")))
    for c in g["cases"]:
        live = np.asarray(c["live"], np.uint8)
        assert int(live.sum()) == c["n_live"]
        s, d = O.plan_compact(live)
        assert s.tolist() == c["src_bt"] and d.tolist() == c["dst_bt"], c
        assert c["src_bt"] == c["movers"] and c["dst_bt"] == c["holes"]


def test_o7_rebalance_worked_examples():
    """The rebalance rule as read (R26) on hand-worked examples
    (tests/golden/r26_rebalance_worked_examples.json): pins the CHOICE of moves — which
    request goes where — not only the plan's invariants."""
    import json, os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "r26_rebalance_worked_examples.json")))
    for c in g["cases"]:
        out, n = O.plan_rebalance(c["n_gpus"], c["req_gpu"], c["req_blocks"])
        assert out.tolist() == c["out_gpu"] and n == c["n_moves"], c
