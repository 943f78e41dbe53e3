"""NEXT-1 with a background mode: pre-pause stages on the copy engines under a rate budget
(wind_kv_migrate_ex), final stage on the TMA kernel; same oracle plan and bytes."""
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


@pytest.mark.parametrize("mode", ["tma_rate", "copy_engines_rate"])
def test_stall_free_background(mode):
    """Background stages at a 200 GB/s budget.  The TMA kernel paces inside the kernel, so
    the decode stream is never held up and the request decodes through several stages.
    The copy-engine mode paces with sleep kernels BETWEEN copies of the migration stream;
    a decode stream that happens to share the migration stream's hardware queue waits
    behind them (CUDA multiplexes streams onto CUDA_DEVICE_MAX_CONNECTIONS queues), so
    only its result is asserted here, not its overlap."""
    sh = SHAPES["C2"]
    bs, T0, capb, nb = sh.block_size, 2048 - 21, 320, 700
    rng = np.random.default_rng(9)
    ss = rng.permutation(nb)[:capb].astype(np.int32)
    ds = rng.permutation(nb)[:capb].astype(np.int32)
    src = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb)
    dst = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, bs, sh.elem_bytes, nb)
    wg.fill(src.base, src.nbytes, 0, 1, 1)
    wg.fill(dst.base, dst.nbytes, 0, 1, 2)
    mig, dec = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
    step = stall_free.append_token_kernel_factory(src, ss, dec)
    st, dt = torch.as_tensor(ss, device=DEV), torch.as_tensor(ds, device=DEV)
    hs, hd = torch.as_tensor(ss).pin_memory(), torch.as_tensor(ds).pin_memory()
    bg = (wk.tuning(kernel=wk.KERNEL_COPY_ENGINE, rate_mbps=200_000) if mode == "copy_engines_rate"
          else wk.tuning(rate_mbps=200_000))  # 200 GB/s budget
    step(T0)
    torch.cuda.synchronize()
    res = stall_free.migrate_stall_free(src, st, dst, dt, T0, 2, step, mig, dec, background=bg,
                                        host_tables=(hs, hd))
    torch.cuda.synchronize()
    want, final = O.stall_free_plan(T0, bs, 2, res.appends + [0] * (64 - len(res.appends)))
    assert res.stages == want and res.final_tokens == final
    if mode == "tma_rate":
        assert len(res.stages) >= 3 and sum(res.appends) > 0, res
    nblk = -(-final // bs)
    S = src.tensor().view(sh.n_layers, 2, nb, -1)
    D = dst.tensor().view(sh.n_layers, 2, nb, -1)
    si = torch.as_tensor(ss[:nblk].astype(np.int64), device=DEV)
    di = torch.as_tensor(ds[:nblk].astype(np.int64), device=DEV)
    for l in range(0, sh.n_layers, 5):
        assert torch.equal(D[l][:, di], S[l][:, si])
    assert all(dst.layer_count(l) == res.ticket for l in range(sh.n_layers))


def test_migrate_ex_rejects_bad_override():
    a = wk.Pool(2, 4, 64, 16, 2, 8)
    b = wk.Pool(2, 4, 64, 16, 2, 8)
    t = torch.arange(4, dtype=torch.int32, device=DEV)
    bad = wk.tuning(stages=2)
    with pytest.raises(wk.WindKVError) as e:
        wk.migrate_ex(a, t, b, t, bad)
    assert e.value.status == -1
    wk.migrate_ex(a, t, b, t, wk.tuning(kernel=wk.KERNEL_SIMT, ctas_per_sm=2, stage_bytes=8192, stages=6))
    torch.cuda.synchronize()
    assert torch.equal(b.tensor().view(2, 2, 8, -1)[:, :, :4], a.tensor().view(2, 2, 8, -1)[:, :, :4])
