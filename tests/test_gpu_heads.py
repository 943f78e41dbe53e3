"""NEXT-3 on the GPU: head-range migrate (TP reshard) and fan-out backups, byte-exact
against the oracle over the whole destination pool."""
import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
from windgen import KVShape

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def geom(p):
    d = p.desc
    return O.Geom(d.first_layer, d.n_layers, d.n_kv_heads, d.head_dim, d.block_size, d.elem_bytes,
                  d.n_blocks)


def rpool(H, nb, seed, L=3, d=128, eb=2):
    p = wk.Pool(L, H, d, 16, eb, nb)
    host = np.random.default_rng(seed).integers(0, 256, p.nbytes, dtype=np.uint8)
    p.tensor().copy_(torch.from_numpy(host))
    return p, host


def tab(a):
    return torch.as_tensor(np.asarray(a, np.int32), device=DEV)


@pytest.fixture(autouse=True)
def default_tuning():
    saved = wk.get_tuning(wk.PATH_INTRA)
    yield
    wk.set_tuning(wk.PATH_INTRA, **saved)


@pytest.mark.parametrize("kernel,unit", [(wk.KERNEL_TMA, 49152), (wk.KERNEL_TMA, 8192),
                                         (wk.KERNEL_SIMT, 32768)])
@pytest.mark.parametrize("Hs,Hd,sh0,dh0,nh", [(8, 4, 4, 0, 4), (4, 8, 0, 4, 4), (8, 8, 2, 5, 3),
                                              (40, 40, 0, 0, 40), (40, 20, 20, 0, 20)])
def test_migrate_heads_matches_oracle(kernel, unit, Hs, Hd, sh0, dh0, nh):
    wk.set_tuning(wk.PATH_INTRA, kernel=kernel, stage_bytes=unit, stages=4)
    src, s0 = rpool(Hs, 70, 1)
    dst, d0 = rpool(Hd, 50, 2)
    rng = np.random.default_rng(Hs * 7 + nh)
    # random entries around a sequential run (coalescible only for whole chunks)
    sp = rng.permutation(np.r_[0:30, 40:70])
    dp = rng.permutation(np.r_[0:5, 15:50])
    sbt = np.concatenate([sp[:10], np.arange(30, 40), sp[10:35]]).astype(np.int32)
    dbt = np.concatenate([dp[:10], np.arange(5, 15), dp[10:35]]).astype(np.int32)
    want = d0.copy()
    assert O.migrate_heads(s0, geom(src), sbt, want, geom(dst), dbt, 1, 3, sh0, dh0, nh) == O.OK
    wk.migrate_heads(src, tab(sbt), dst, tab(dbt), sh0, dh0, nh, layer_lo=1, layer_hi=3)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(dst.tensor().cpu().numpy(), want)


def test_tp2_to_tp1_reshard_on_gpu():
    """[TP-2, TP-1] (Fig. 3): two prefill shards push their head halves into one
    decode pool; equals a direct migration of the unsharded KV."""
    H = 40
    full, f0 = rpool(H, 64, 3)
    shards = []
    F = f0.reshape(3, 2, 64, H, -1)
    for r in range(2):
        p = wk.Pool(3, H // 2, 128, 16, 2, 64)
        p.tensor().copy_(torch.from_numpy(np.ascontiguousarray(F[:, :, :, r * 20:(r + 1) * 20]).reshape(-1)))
        shards.append(p)
    dec, e0 = rpool(H, 80, 4)
    ref, _ = rpool(H, 80, 4)
    sbt = np.random.default_rng(0).permutation(64)[:33].astype(np.int32)
    dbt = np.random.default_rng(1).permutation(80)[:33].astype(np.int32)
    for r in range(2):
        wk.migrate_heads(shards[r], tab(sbt), dec, tab(dbt), 0, r * 20, 20)
    wk.migrate(full, tab(sbt), ref, tab(dbt))
    torch.cuda.synchronize()
    assert torch.equal(dec.tensor(), ref.tensor())
    assert dec.layer_ticket() == 2 and dec.layer_count(0) == 2


def test_fanout_backup_two_destinations():
    """NEXT-3 backups: one source block set copied to two pools in ONE launch
    (duplicate sources across items = fan-out)."""
    src, s0 = rpool(8, 60, 5)
    a, a0 = rpool(8, 40, 6)
    b, b0 = rpool(8, 45, 7)
    sbt = np.random.default_rng(2).permutation(60)[:30].astype(np.int32)
    da = np.random.default_rng(3).permutation(40)[:30].astype(np.int32)
    db = np.random.default_rng(4).permutation(45)[:30].astype(np.int32)
    wk.migrate_batch(src, [(a, tab(sbt), tab(da)), (b, tab(sbt), tab(db))], 0, 3)
    torch.cuda.synchronize()
    for pool, p0, d in ((a, a0, da), (b, b0, db)):
        want = p0.copy()
        assert O.migrate(s0, geom(src), sbt, want, geom(pool), d, 0, 3) == O.OK
        np.testing.assert_array_equal(pool.tensor().cpu().numpy(), want)


def test_heads_errors_match_oracle():
    a, _ = rpool(8, 10, 1)
    b, _ = rpool(4, 10, 2)
    c = wk.Pool(3, 4, 64, 16, 2, 10)
    for args, (s0, d0, nh) in [((a, b), (4, 0, 4)), ((a, b), (4, 1, 4)), ((a, b), (6, 0, 4)),
                               ((a, b), (0, 0, 0)), ((a, c), (0, 0, 2))]:
        try:
            wk.migrate_heads(args[0], tab([1]), args[1], tab([2]), s0, d0, nh)
            got = 0
        except wk.WindKVError as e:
            got = e.status
        assert got == O.check_op_heads(geom(args[0]), geom(args[1]), 1, 0, 3, s0, d0, nh)
    torch.cuda.synchronize()


@pytest.mark.parametrize("k", [2, 3, 4, 5])
@pytest.mark.parametrize("unit,stages", [(49152, 4), (8192, 6), (65536, 3)])
@pytest.mark.parametrize("H", [8, 1])
def test_read_once_fanout(k, unit, stages, H):
    """NEXT-3 backups, read-once: every batch item passes the SAME source table, so the TMA
    kernel stages each source unit once and stores it to all k destinations (k <= 4; k = 5
    takes the per-item path).  Mixed destination tables (one sequential, others shuffled)
    break runs in some destinations only; whole pools + flags vs the oracle."""
    wk.set_tuning(wk.PATH_INTRA, kernel=wk.KERNEL_TMA, stage_bytes=unit, stages=stages)
    rng = np.random.default_rng(100 + k)
    nb = 90
    src, s0 = rpool(H, nb, 50)          # C = 32 KiB (parts / 1-2 per unit) or 4 KiB (windows of 16)
    n = 61
    sbt = np.sort(rng.permutation(nb)[:n]).astype(np.int32)   # long source runs
    sbt[::7] = rng.integers(0, nb, sbt[::7].size)              # ... broken, with duplicates
    ts = tab(sbt)                                              # ONE table object for all items
    dsts = []
    for j in range(k):
        d, d0 = rpool(H, nb + 3 * j, 60 + j)
        db = (np.arange(n) + j) if j == 0 else rng.permutation(nb + 3 * j)[:n]
        dsts.append((d, d0, db.astype(np.int32)))
    n0 = wk.launch_count()
    wk.migrate_batch(src, [(d, ts, tab(db)) for d, _, db in dsts], 1, 3)
    torch.cuda.synchronize()
    assert wk.launch_count() - n0 == 1
    for d, d0, db in dsts:
        want = d0.copy()
        assert O.migrate(s0, geom(src), sbt, want, geom(d), db, 1, 3) == O.OK
        np.testing.assert_array_equal(d.tensor().cpu().numpy(), want)
        assert d.layer_ticket() == 1 and [d.layer_count(l) for l in range(3)] == [1, 1, 1]
