"""GPU: the copy-engine path (tuning kernel = 3) — TP head ranges, batches, the rate limit,
and its flag publication."""
import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
import windgen.cuda as wg
from windgen import SHAPES

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def geom(p):
    d = p.desc
    return O.Geom(d.first_layer, d.n_layers, d.n_kv_heads, d.head_dim, d.block_size, d.elem_bytes,
                  d.n_blocks)


@pytest.fixture(autouse=True)
def ce_tuning():
    saved = wk.get_tuning(wk.PATH_INTRA)
    wk.set_tuning(wk.PATH_INTRA, **{**saved, "kernel": wk.KERNEL_COPY_ENGINE})
    yield
    wk.set_tuning(wk.PATH_INTRA, **saved)


def rpool(H, nb, seed, L=3):
    p = wk.Pool(L, H, 128, 16, 2, nb)
    h = np.random.default_rng(seed).integers(0, 256, p.nbytes, dtype=np.uint8)
    p.tensor().copy_(torch.from_numpy(h))
    return p, h


def htab(a):
    return torch.as_tensor(np.asarray(a, np.int32)).pin_memory()


def test_ce_heads_and_runs():
    src, s0 = rpool(8, 70, 1)
    dst, d0 = rpool(4, 50, 2)
    sbt = np.r_[np.arange(30, 40), [3, 9, 61]].astype(np.int32)
    dbt = np.r_[np.arange(5, 15), [40, 2, 30]].astype(np.int32)
    want = d0.copy()
    assert O.migrate_heads(s0, geom(src), sbt, want, geom(dst), dbt, 1, 3, 4, 0, 4) == O.OK
    hs, hd = htab(sbt), htab(dbt)
    wk.migrate_heads(src, hs.data_ptr(), dst, hd.data_ptr(), 4, 0, 4, n=len(sbt), layer_lo=1, layer_hi=3)
    torch.cuda.synchronize()
    np.testing.assert_array_equal(dst.tensor().cpu().numpy(), want)
    assert [dst.layer_count(l) for l in range(3)] == [1, 1, 1]


def test_ce_batch_two_destinations():
    src, s0 = rpool(8, 60, 3)
    a, a0 = rpool(8, 40, 4)
    b, b0 = rpool(8, 45, 5)
    sbt = np.random.default_rng(0).permutation(60)[:20].astype(np.int32)
    da = np.random.default_rng(1).permutation(40)[:20].astype(np.int32)
    db = np.random.default_rng(2).permutation(45)[:20].astype(np.int32)
    keep = [htab(sbt), htab(da), htab(db)]
    wk.migrate_batch(src, [(a, keep[0].data_ptr(), keep[1].data_ptr(), 20),
                           (b, keep[0].data_ptr(), keep[2].data_ptr(), 20)], 0, 3)
    torch.cuda.synchronize()
    for pool, p0, d in ((a, a0, da), (b, b0, db)):
        want = p0.copy()
        assert O.migrate(s0, geom(src), sbt, want, geom(pool), d, 0, 3) == O.OK
        np.testing.assert_array_equal(pool.tensor().cpu().numpy(), want)


def test_ce_rate_limit():
    sh = SHAPES["C2"]
    nb = 300
    src = wk.Pool(4, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
    dst = wk.Pool(4, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
    wg.fill(src.base, src.nbytes, 0, 1, 1)
    sbt = htab(np.random.default_rng(0).permutation(nb)[:256])
    dbt = htab(np.random.default_rng(1).permutation(nb)[:256])
    payload = 2 * 4 * 256 * sh.chunk_bytes
    s = torch.cuda.Stream(DEV)
    saved = wk.get_tuning(wk.PATH_INTRA)
    for rate in (50, 200):
        wk.set_tuning(wk.PATH_INTRA, **{**saved, "rate_mbps": rate * 1000})
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        wk.migrate(src, sbt.data_ptr(), dst, dbt.data_ptr(), n=256, stream=s)
        b.record(s)
        torch.cuda.synchronize()
        got = payload / (a.elapsed_time(b) * 1e6)
        assert 0.8 * rate < got < 1.1 * rate, (rate, got)
    S = src.tensor().view(4, 2, nb, -1)
    D = dst.tensor().view(4, 2, nb, -1)
    assert torch.equal(D[:, :, dbt.long().to(DEV)], S[:, :, sbt.long().to(DEV)])
