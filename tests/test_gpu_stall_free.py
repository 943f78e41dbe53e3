"""NEXT-1: stall-free multi-stage migration on the GPU, pinned to the oracle's O8
plan (the stages) and to the oracle's O3 migrate run on the SOURCE POOL AT THE PAUSE (P9):
the whole destination pool — every layer, K and V, untouched slots included — must equal
what O3 makes of the initial destination with the source as it stood when decoding paused.
(Full blocks are immutable and the request's last block is only sent after the pause, so
the staged migration must reach exactly that state.)"""
import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
from paper_conf_isca_fenghzly025_b200 import stall_free
import windgen.cuda as wg
from windgen import SHAPES

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


@pytest.mark.parametrize("theta,cap,chunk", [(2, 2, 0), (1, 4, 0), (8, 0, 0), (2, 0, 8), (1, 0, 3)])
def test_stall_free_migration_matches_oracle(theta, cap, chunk):
    """P:120's request: OPT-13B KV, 2048 tokens (1.5625 GiB).  The migration is throttled
    (CTA cap) so the request decodes through several stages; with `chunk`, each stage is
    issued as one burst of `chunk` blocks per decode step (full rate)."""
    sh = SHAPES["C2"]
    bs = sh.block_size
    T0 = 2048 - 37
    cap_blocks = 320
    nb = 400  # 5 GiB per pool: both pools are compared whole against the oracle
    rng = np.random.default_rng(theta)
    src_slots = rng.permutation(nb)[:cap_blocks].astype(np.int32)
    dst_slots = rng.permutation(nb)[:cap_blocks].astype(np.int32)
    src = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb)
    dst = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb)
    wg.fill(src.base, src.nbytes, 0, 1, 1)
    wg.fill(dst.base, dst.nbytes, 0, 1, 2)
    torch.cuda.synchronize()
    d0 = dst.tensor().cpu().numpy()  # destination before the migration
    saved = wk.get_tuning(wk.PATH_INTRA)
    wk.set_tuning(wk.PATH_INTRA, **{**saved, "max_ctas": cap})
    try:
        mig, dec = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
        step = stall_free.append_token_kernel_factory(src, src_slots, dec)
        st = torch.as_tensor(src_slots, device=DEV)
        dt = torch.as_tensor(dst_slots, device=DEV)
        step(T0)  # warm the append kernel (idempotent: the same bytes are written again later)
        torch.cuda.synchronize()
        res = stall_free.migrate_stall_free(src, st, dst, dt, T0, theta, step, mig, dec, chunk_blocks=chunk)
    finally:
        wk.set_tuning(wk.PATH_INTRA, **saved)
    torch.cuda.synchronize()
    # the plan the driver followed is the oracle's plan for the appends that happened
    want, final = O.stall_free_plan(T0, bs, theta, res.appends + [0] * (64 - len(res.appends)))
    assert res.stages == want and res.final_tokens == final
    assert sum(res.appends) >= len(res.appends) >= 1  # decoding continued during migration
    nblk = -(-final // bs)
    assert res.blocks_sent == nblk  # every block sent exactly once
    # the oracle's O3 on the source at the pause (decoding paused before the final stage and
    # never resumed on the source), applied to the initial destination, whole pools
    s_pause = src.tensor().cpu().numpy()
    gs = O.Geom(0, sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb)
    want = d0.copy()
    assert O.migrate(s_pause, gs, src_slots[:nblk], want, gs, dst_slots[:nblk], 0, sh.n_layers) == O.OK
    got = dst.tensor().cpu().numpy()
    if not np.array_equal(got, want):
        bad = np.flatnonzero((got != want).reshape(sh.n_layers, 2, nb, -1).any(axis=-1))
        l, kv, b = np.unravel_index(bad[0], (sh.n_layers, 2, nb))
        raise AssertionError(f"{bad.size} chunks differ from the oracle; first: layer {l} kv {kv} slot {b}")
    # the appends really changed the source during the migration (the pin is not vacuous):
    # the last block sent holds tokens written after T0
    assert sum(res.appends) > 0
    assert all(dst.layer_count(l) == res.ticket for l in range(sh.n_layers))
    if theta < 8:  # capped: the request outgrows theta during stage 0; bursts: at least one stage + pause
        assert len(res.stages) >= (2 if chunk else 3)
    if chunk:  # every pre-pause stage took at least one decode step per burst
        for (b, e), a in zip(res.stages[:-1], res.appends):
            assert a >= -(-(e - b) // chunk)
