"""NEXT-4 on the GPU path: the Dynamic Rescheduling trigger and victim policy (host logic,
``policy.py``; "when the KV blocks of decoding instances are nearly
exhausted ... rescheduling long-context requests", P:233 longest first; readings R7, R8,
R10) driving a real decode -> prefill migration through the C ABI, checked against the
oracle.

A decode pool at 97.5 % occupancy fires the trigger; the victims (longest first) are moved
to the prefill instance's pool into its lowest free slots in ONE migrate; the whole prefill
pool must equal oracle O3's result, every victim's logical KV (read through its new block
table) must equal what it was in the decode pool, and the freed decode blocks must cover
the deficit the policy was asked to clear.
"""
import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
from paper_conf_isca_fenghzly025_b200 import policy
from windgen import SHAPES

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def geom(p: wk.Pool) -> O.Geom:
    d = p.desc
    return O.Geom(d.first_layer, d.n_layers, d.n_kv_heads, d.head_dim, d.block_size, d.elem_bytes,
                  d.n_blocks)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_trigger_victims_and_migration_match_oracle(seed):
    sh = SHAPES["C1"]                      # OPT-125M KV: 12 layers, C = 24 KiB
    bs = sh.block_size
    rng = np.random.default_rng(seed)
    nb_dec, nb_pre = 200, 160
    # decode instance: requests with ShareGPT-like lengths packed into a shuffled pool
    lens = []
    while sum(-(-t // bs) for t in lens) < 195:
        lens.append(int(rng.integers(40, 900)))
    blocks = [-(-t // bs) for t in lens]
    over = sum(blocks) - 195
    blocks[-1] -= over                     # exactly 195 live blocks (97.5 %)
    lens[-1] = blocks[-1] * bs
    perm = rng.permutation(nb_dec).astype(np.int32)
    starts = np.concatenate([[0], np.cumsum(blocks)])
    tables = [perm[starts[r]:starts[r + 1]] for r in range(len(blocks))]
    free_dec = nb_dec - int(starts[-1])
    new_per_step = sum(1 for t in lens if t % bs == 0)  # requests whose next token opens a block
    assert policy.should_reschedule(free_dec, nb_dec, new_per_step)
    need = int(np.ceil(0.2 * nb_dec)) - free_dec       # free 20 % of the pool
    victims = policy.pick_victims(blocks, need)
    assert sum(blocks[r] for r in victims) >= need
    order = sorted(range(len(blocks)), key=lambda r: (-blocks[r], r))
    assert victims == order[:len(victims)]              # longest first (R7)

    dec = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb_dec)
    pre = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb_pre)
    d0 = rng.integers(0, 256, dec.nbytes, dtype=np.uint8)
    p0 = rng.integers(0, 256, pre.nbytes, dtype=np.uint8)
    dec.tensor().copy_(torch.from_numpy(d0))
    pre.tensor().copy_(torch.from_numpy(p0))
    # prefill instance: 30 % of its slots busy; victims land lowest-free-first (R10)
    busy = rng.random(nb_pre) < 0.3
    free_pre = np.flatnonzero(~busy).astype(np.int32)
    src_bt = np.concatenate([tables[r] for r in victims]).astype(np.int32)
    assert src_bt.size <= free_pre.size
    dst_bt = free_pre[:src_bt.size]
    assert wk.validate(dec, src_bt, pre, dst_bt, 0, sh.n_layers) == 0
    wk.migrate(dec, torch.as_tensor(src_bt, device=DEV), pre, torch.as_tensor(dst_bt, device=DEV))
    torch.cuda.synchronize()
    want = p0.copy()
    assert O.migrate(d0, geom(dec), src_bt, want, geom(pre), dst_bt, 0, sh.n_layers) == O.OK
    got = pre.tensor().cpu().numpy()
    np.testing.assert_array_equal(got, want)
    # each victim's logical KV through its new table == its KV in the decode pool
    new_tables, k = {}, 0
    for r in victims:
        new_tables[r] = dst_bt[k:k + blocks[r]]
        k += blocks[r]
    D = d0.reshape(sh.n_layers, 2, nb_dec, -1)
    P = got.reshape(sh.n_layers, 2, nb_pre, -1)
    for r in victims:
        np.testing.assert_array_equal(P[:, :, new_tables[r]], D[:, :, tables[r]])
    assert free_dec + int(src_bt.size) >= int(np.ceil(0.2 * nb_dec))
    assert [pre.layer_count(l) for l in range(sh.n_layers)] == [1] * sh.n_layers
