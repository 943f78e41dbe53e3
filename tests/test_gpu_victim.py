"""The interference victim (bench harness, not the product): paged decode attention over a
wind_kv pool, checked against plain PyTorch fp32 attention (SDPA definition)."""
import math

import numpy as np
import pytest
import torch

import paper_conf_isca_fenghzly025_b200 as wk
import victim

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


@pytest.mark.parametrize("hq,hkv", [(8, 8), (8, 2)])
def test_victim_matches_torch_attention(hq, hkv):
    L, bs, d = 3, 16, 128
    lens = [37, 100, 16, 513]
    B = len(lens)
    nb = 80
    pool = wk.Pool(L, hkv, d, bs, 2, nb)
    pt = pool.tensor().view(torch.float16)
    torch.manual_seed(0)
    pt.copy_(torch.randn(pt.numel(), device=DEV, dtype=torch.float16))
    max_blocks = max(-(-n // bs) for n in lens)
    rng = np.random.default_rng(1)
    slots = rng.permutation(nb)
    bt = np.zeros((B, max_blocks), np.int32)
    pos = 0
    for b, n in enumerate(lens):
        k = -(-n // bs)
        bt[b, :k] = slots[pos:pos + k]
        pos += k
    bt_t = torch.as_tensor(bt, device=DEV)
    ctx = torch.as_tensor(np.array(lens, np.int32), device=DEV)
    q = torch.randn(B, hq, d, device=DEV, dtype=torch.float16)
    layer = 1
    plane = nb * hkv * bs * d * 2
    kp = pool.base + (layer * 2 + 0) * plane
    vp = pool.base + (layer * 2 + 1) * plane
    scratch = torch.empty(victim.scratch_floats(B, hq, max_blocks, 2), device=DEV)
    out = torch.empty(B, hq, d, device=DEV)
    victim.decode_attention(q, kp, vp, bt_t, ctx, hkv, bs, scratch, out, blocks_per_split=2)
    torch.cuda.synchronize()
    P = pt.view(L, 2, nb, hkv, bs, d).float()
    for b, n in enumerate(lens):
        k = -(-n // bs)
        K = P[layer, 0, bt[b, :k]].permute(1, 0, 2, 3).reshape(hkv, k * bs, d)[:, :n]
        V = P[layer, 1, bt[b, :k]].permute(1, 0, 2, 3).reshape(hkv, k * bs, d)[:, :n]
        for h in range(hq):
            kh = h // (hq // hkv)
            s = (q[b, h].float() @ K[kh].T) / math.sqrt(d)
            ref = torch.softmax(s, dim=0) @ V[kh]
            torch.testing.assert_close(out[b, h], ref, rtol=2e-3, atol=2e-3)
