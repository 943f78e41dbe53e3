"""NEXT-2: layer-streamed prefill -> decode hand-off overlapped with a running prefill
(§1 "overlapping KV transfers with prefill computations", §5.2; S§8(f)).

A synthetic OPT-13B-shaped prefill (bf16 GEMMs on the prefill stream) computes layer l and
WRITES that layer's K and V of the request into the source pool (the GEMM outputs' bytes);
an event recorded after layer l releases migrate(layer l, l + 1) on a side stream, and a
consumer stream waits on the destination's layer_done[l] with that op's ticket
(wind_kv_layer_wait), then snapshots layer l of the destination.  Pinned to the oracle:

  * the whole destination pool equals O3 (oracle.migrate, all layers) applied to its initial
    bytes with the source as the prefill left it — every layer's K/V came from the prefill,
    so a migration that ran ahead of its event would copy stale bytes and fail;
  * every consumer snapshot of layer l already holds the oracle's layer l (the flag never
    moves before its layer's bytes);
  * ticket of op l = l + 1, and every destination layer flag ends at L (R23: each op bumps
    every destination layer exactly once).
"""
import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
from windgen import SHAPES

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


@pytest.fixture(autouse=True)
def default_tuning():
    saved = {p: wk.get_tuning(p) for p in (wk.PATH_INTRA, wk.PATH_PEER, wk.PATH_HOST)}
    yield
    for p, t in saved.items():
        wk.set_tuning(p, **t)


def geom(p: wk.Pool) -> O.Geom:
    d = p.desc
    return O.Geom(d.first_layer, d.n_layers, d.n_kv_heads, d.head_dim, d.block_size, d.elem_bytes,
                  d.n_blocks)


@pytest.mark.parametrize("kernel,cap", [(wk.KERNEL_TMA, 16), (wk.KERNEL_TMA, 0), (wk.KERNEL_SIMT, 8)])
def test_prefill_overlapped_handoff_matches_oracle(kernel, cap):
    sh = SHAPES["C2"]                       # 40 layers, 40 heads, d = 128, fp16: C = 160 KiB
    L, bs, C = sh.n_layers, sh.block_size, sh.chunk_bytes
    H = sh.n_kv_heads * sh.head_dim         # hidden size 5120
    n_tokens = 512                          # 32 blocks: one layer's K (or V) = 512 x 5120 bf16
    nblk = n_tokens // bs
    nb_src, nb_dst = nblk + 9, nblk + 17
    rng = np.random.default_rng(kernel * 100 + cap)
    sbt = rng.permutation(nb_src)[:nblk].astype(np.int32)
    dbt = rng.permutation(nb_dst)[:nblk].astype(np.int32)
    src = wk.Pool(L, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb_src)
    dst = wk.Pool(L, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb_dst)
    s_init = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
    d0 = rng.integers(0, 256, dst.nbytes, dtype=np.uint8)
    src.tensor().copy_(torch.from_numpy(s_init))
    dst.tensor().copy_(torch.from_numpy(d0))
    wk.set_tuning(wk.PATH_INTRA, kernel=kernel, max_ctas=cap)

    g = torch.Generator(device=DEV).manual_seed(7)
    x = torch.randn(n_tokens, H, device=DEV, dtype=torch.bfloat16, generator=g)
    w_k = torch.randn(H, H, device=DEV, dtype=torch.bfloat16, generator=g) * 0.02
    w_v = torch.randn(H, H, device=DEV, dtype=torch.bfloat16, generator=g) * 0.02
    w_o = torch.randn(H, H, device=DEV, dtype=torch.bfloat16, generator=g) * 0.02
    sview = src.tensor().view(L, 2, nb_src, C)
    dview = dst.tensor().view(L, 2, nb_dst, C)
    s_idx = torch.as_tensor(sbt.astype(np.int64), device=DEV)
    d_idx = torch.as_tensor(dbt.astype(np.int64), device=DEV)
    st, dt = torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV)
    snaps = torch.empty(L, 2, nblk, C, dtype=torch.uint8, device=DEV)
    pre, mig, cons = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
    torch.cuda.synchronize()

    tickets = []
    keep = []  # prefill outputs stay alive until the streams are joined
    h = x
    for l in range(L):
        with torch.cuda.stream(pre):  # prefill layer l: its K and V land in the source pool
            k = h @ w_k
            v = h @ w_v
            sview[l, 0, s_idx] = k.view(torch.uint8).view(nblk, C)
            sview[l, 1, s_idx] = v.view(torch.uint8).view(nblk, C)
            h = torch.tanh(h @ w_o)
            keep += [k, v, h]
        ev = torch.cuda.Event()
        ev.record(pre)
        mig.wait_event(ev)
        wk.migrate(src, st, dst, dt, layer_lo=l, layer_hi=l + 1, stream=mig)
        t = dst.layer_ticket()
        tickets.append(t)
        wk.layer_wait(dst, l, t, stream=cons)  # the decode side picks layer l up as it lands
        with torch.cuda.stream(cons):
            snaps[l] = dview[l][:, d_idx]
    torch.cuda.synchronize()
    assert tickets == list(range(1, L + 1))

    s_final = src.tensor().cpu().numpy()
    want = d0.copy()
    assert O.migrate(s_final, geom(src), sbt, want, geom(dst), dbt, 0, L) == O.OK
    got = dst.tensor().cpu().numpy()
    np.testing.assert_array_equal(got, want)
    # the prefill really produced the migrated bytes (the pin is not vacuous)
    assert not np.array_equal(s_final, s_init)
    w4 = want.reshape(L, 2, nb_dst, C)[:, :, dbt]
    np.testing.assert_array_equal(snaps.cpu().numpy(), w4)
    assert [dst.layer_count(l) for l in range(L)] == [L] * L
    assert [src.layer_count(l) for l in range(L)] == [0] * L
