"""NEXT-1: stall-free multi-stage migration on the GPU, pinned to the oracle's O8
plan and to the source content at the pause (P9)."""
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


@pytest.mark.parametrize("theta,cap", [(2, 2), (1, 4), (8, 0)])
def test_stall_free_migration_matches_oracle(theta, cap):
    """P:120's request: OPT-13B KV, 2048 tokens (1.5625 GiB).  The migration is throttled
    (CTA cap) so the request decodes through several stages."""
    sh = SHAPES["C2"]
    bs = sh.block_size
    T0 = 2048 - 37
    cap_blocks = 320
    nb = 700
    rng = np.random.default_rng(theta)
    src_slots = rng.permutation(nb)[:cap_blocks].astype(np.int32)
    dst_slots = rng.permutation(nb)[:cap_blocks].astype(np.int32)
    src = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb)
    dst = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb)
    wg.fill(src.base, src.nbytes, 0, 1, 1)
    wg.fill(dst.base, dst.nbytes, 0, 1, 2)
    saved = wk.get_tuning(wk.PATH_INTRA)
    wk.set_tuning(wk.PATH_INTRA, **{**saved, "max_ctas": cap})
    try:
        mig, dec = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
        step = stall_free.append_token_kernel_factory(src, src_slots, dec)
        st = torch.as_tensor(src_slots, device=DEV)
        dt = torch.as_tensor(dst_slots, device=DEV)
        step(T0)  # warm the append kernel (idempotent: the same bytes are written again later)
        torch.cuda.synchronize()
        res = stall_free.migrate_stall_free(src, st, dst, dt, T0, theta, step, mig, dec)
    finally:
        wk.set_tuning(wk.PATH_INTRA, **saved)
    torch.cuda.synchronize()
    # the plan the driver followed is the oracle's plan for the appends that happened
    want, final = O.stall_free_plan(T0, bs, theta, res.appends + [0] * (64 - len(res.appends)))
    assert res.stages == want and res.final_tokens == final
    assert sum(res.appends) >= len(res.appends) >= 1  # decoding continued during migration
    nblk = -(-final // bs)
    assert res.blocks_sent == nblk  # every block sent exactly once
    # destination == source at the pause, every layer, K and V, whole blocks
    S = src.tensor().view(sh.n_layers, 2, nb, -1)
    D = dst.tensor().view(sh.n_layers, 2, nb, -1)
    for l in range(0, sh.n_layers, 7):
        assert torch.equal(D[l][:, torch.as_tensor(dst_slots[:nblk].astype(np.int64), device=DEV)],
                           S[l][:, torch.as_tensor(src_slots[:nblk].astype(np.int64), device=DEV)])
    assert all(dst.layer_count(l) == res.ticket for l in range(sh.n_layers))
    if theta < 8:
        assert len(res.stages) >= 3
