"""GPU: release builds never touch memory outside the two pools, even with a bad table.

include/wind_kv.h (migrate, "Table contract"): release builds do not CHECK table content on
the hot path (WIND_POOL_DEBUG pools and wind_kv_validate do), but an entry outside
[0, NB) of its pool is skipped by the copy kernels — no byte of it is read or written.
These tests put pools inside larger allocations with canary guards on both sides and pass
tables with entries just outside the pool (NB, NB + 1, -1: unguarded, those addresses land
in the guards or in a neighbouring plane of the same allocation, so a broken guard shows
up as changed bytes, never as a fault).  Expected: the whole destination pool equals the
oracle's migrate of the VALID entries only, both canaries are intact, and every layer flag
still moves once (a consumer waiting on the op's ticket is released).
"""
import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)
GUARD = 1 << 20  # bytes of canary before and after each pool (>= 2 chunks at every geometry here)


def guarded_pool(L, H, d, bs, eb, nb, seed):
    """A pool over the middle of a torch buffer; returns (pool, buffer, pool bytes)."""
    C = H * d * bs * eb
    pbytes = L * 2 * nb * C
    g = torch.Generator().manual_seed(seed)
    buf = torch.randint(0, 256, (GUARD + pbytes + GUARD,), dtype=torch.uint8, generator=g).to(DEV)
    pool = wk.Pool(L, H, d, bs, eb, nb, external_base=buf.data_ptr() + GUARD)
    return pool, buf, pbytes


def geom(L, H, d, bs, eb, nb):
    return O.Geom(0, L, H, d, bs, eb, nb)


TUNINGS = {"tma": None,
           "simt": lambda: wk.tuning(kernel=wk.KERNEL_SIMT, stage_bytes=32768, stages=4)}


@pytest.mark.parametrize("kern", sorted(TUNINGS))
@pytest.mark.parametrize("H", [8, 16])  # 32 KiB chunks (run windows) / 64 KiB (split into parts)
def test_out_of_range_entries_are_skipped(kern, H):
    L, d, bs, eb = 3, 128, 16, 2
    nbs, nbd = 40, 36
    src, sbuf, sb = guarded_pool(L, H, d, bs, eb, nbs, 1)
    dst, dbuf, db = guarded_pool(L, H, d, bs, eb, nbd, 2)
    s_all = sbuf.cpu().numpy()
    d_all = dbuf.cpu().numpy()
    # valid runs (coalescable 5..9 -> 10..14), broken by bad entries on either side
    sbt = np.array([5, 6, nbs, 7, 8, 9, -1, 20, 21, 22, 3, nbs + 1, 30, 31], np.int32)
    dbt = np.array([10, 11, 12, nbd, 14, 15, 16, 17, -1, 19, 0, 1, nbd + 1, 35], np.int32)
    ok = (sbt >= 0) & (sbt < nbs) & (dbt >= 0) & (dbt < nbd)
    ts, td = torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV)
    t = TUNINGS[kern]() if TUNINGS[kern] else None
    wk.migrate_ex(src, ts, dst, td, t)
    torch.cuda.synchronize()
    got = dbuf.cpu().numpy()
    want = d_all[GUARD:GUARD + db].copy()
    assert O.migrate(s_all[GUARD:GUARD + sb], geom(L, H, d, bs, eb, nbs), sbt[ok], want,
                     geom(L, H, d, bs, eb, nbd), dbt[ok], 0, L) == O.OK
    np.testing.assert_array_equal(got[:GUARD], d_all[:GUARD])                 # canary before
    np.testing.assert_array_equal(got[GUARD + db:], d_all[GUARD + db:])       # canary after
    np.testing.assert_array_equal(got[GUARD:GUARD + db], want)
    np.testing.assert_array_equal(sbuf.cpu().numpy(), s_all)                  # source untouched
    assert dst.layer_ticket() == 1 and [dst.layer_count(l) for l in range(L)] == [1] * L


def test_fan_out_skips_an_entry_bad_in_any_destination():
    """Read-once fan-out (one source table, two destinations): an entry out of range in
    EITHER destination is skipped for both; the others land in both pools."""
    L, H, d, bs, eb = 2, 8, 128, 16, 2
    nb = 24
    src, sbuf, sb = guarded_pool(L, H, d, bs, eb, nb, 3)
    a, abuf, ab = guarded_pool(L, H, d, bs, eb, nb, 4)
    b, bbuf, bb = guarded_pool(L, H, d, bs, eb, nb, 5)
    s_all, a_all, b_all = sbuf.cpu().numpy(), abuf.cpu().numpy(), bbuf.cpu().numpy()
    sbt = np.array([0, 1, 2, 3, 4, 5, 6], np.int32)
    dba = np.array([7, 8, nb, 10, 11, -1, 13], np.int32)
    dbb = np.array([2, 3, 4, nb + 1, 6, 9, 8], np.int32)
    ok = (dba >= 0) & (dba < nb) & (dbb >= 0) & (dbb < nb)
    ts = torch.as_tensor(sbt, device=DEV)  # ONE source table object: the fan-out path
    wk.migrate_batch(src, [(a, ts, torch.as_tensor(dba, device=DEV)), (b, ts, torch.as_tensor(dbb, device=DEV))], 0, L)
    torch.cuda.synchronize()
    g = geom(L, H, d, bs, eb, nb)
    for buf, full, nbytes, dbt in ((abuf, a_all, ab, dba), (bbuf, b_all, bb, dbb)):
        got = buf.cpu().numpy()
        want = full[GUARD:GUARD + nbytes].copy()
        assert O.migrate(s_all[GUARD:GUARD + sb], g, sbt[ok], want, g, dbt[ok], 0, L) == O.OK
        np.testing.assert_array_equal(got[:GUARD], full[:GUARD])
        np.testing.assert_array_equal(got[GUARD + nbytes:], full[GUARD + nbytes:])
        np.testing.assert_array_equal(got[GUARD:GUARD + nbytes], want)
    assert [a.layer_count(l) for l in range(L)] == [1] * L
    assert [b.layer_count(l) for l in range(L)] == [1] * L


def test_all_entries_out_of_range_still_publishes():
    """Nothing valid: no byte moves, and every layer flag still moves once."""
    L, H, d, bs, eb = 4, 8, 128, 16, 2
    nb = 16
    src, sbuf, _ = guarded_pool(L, H, d, bs, eb, nb, 6)
    dst, dbuf, _ = guarded_pool(L, H, d, bs, eb, nb, 7)
    d_all = dbuf.cpu().numpy()
    sbt = np.array([nb, -1, nb + 1], np.int32)
    dbt = np.array([0, 1, 2], np.int32)
    wk.migrate(src, torch.as_tensor(sbt, device=DEV), dst, torch.as_tensor(dbt, device=DEV))
    torch.cuda.synchronize()
    np.testing.assert_array_equal(dbuf.cpu().numpy(), d_all)
    assert [dst.layer_count(l) for l in range(L)] == [1] * L
