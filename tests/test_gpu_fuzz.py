"""GPU parity fuzz: random pool geometries, tables, layer windows, head ranges and launch
tunings, each op compared with the CPU oracle over the WHOLE destination pool and its
layer flags (readings R3-R5, R19-R24).

What a fixed-shape test can miss and this one draws at random: chunk sizes C that are not
a multiple of the work unit (ragged parts, ragged windows), units smaller than one chunk
or holding up to 32 chunks, 1-16 token blocks, fp8 / fp16 / fp32 elements, pools whose
layer windows are shifted (PP stages, `first_layer`), empty and one-block tables, duplicate
sources (fan-out), same-pool moves with identity pairs, host pools (swap), grids capped
below the unit count, ring depths 3-8 with every store lag, the copy-engine path, and
(round 2) burst-paced ops and step-released slices (wind_kv_migrate_stepped) of the
two-pool moves.
"""
import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)
N_CASES = 400


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


def filled(rng, L, H, d, bs, eb, nb, first, loc="device"):
    p = wk.Pool(L, H, d, bs, eb, nb, loc=loc, first_layer=first)
    host = rng.integers(0, 256, p.nbytes, dtype=np.uint8)
    p.tensor().copy_(torch.from_numpy(host))
    return p, host


def read(p: wk.Pool) -> np.ndarray:
    torch.cuda.synchronize()
    return p.tensor().cpu().numpy().copy()


def draw_tuning(rng, kernel):
    if kernel in (wk.KERNEL_COPY_ENGINE, wk.KERNEL_STAGED):
        return dict(kernel=kernel, stage_bytes=32768, stages=4)
    unit = int(rng.choice([16, 48, 256, 2048, 4096, 12288, 32768, 49152, 131072]))
    if kernel == wk.KERNEL_TMA:
        unit = min(unit, 49152)
        stages = int(rng.integers(3, 9))
        while stages * unit > 200 * 1024:
            stages -= 1
        stages = max(stages, 3)
        lag = int(rng.integers(0, stages))
    else:
        stages, lag = 4, 0
    return dict(kernel=kernel, stage_bytes=unit, stages=stages, store_lag=lag,
                ctas_per_sm=int(rng.integers(1, 3)), max_ctas=int(rng.choice([0, 0, 1, 3, 17])))


@pytest.mark.parametrize("seed", range(N_CASES))
def test_random_op_matches_oracle(seed):
    rng = np.random.default_rng(10_000 + seed)
    eb = int(rng.choice([1, 2, 4]))
    d = int(rng.choice([16, 32, 64, 80, 128]))       # d * eb % 16 == 0 for every eb
    H = int(rng.integers(1, 7))
    bs = int(rng.choice([1, 2, 4, 16]))
    Ls, Ld = int(rng.integers(1, 7)), int(rng.integers(1, 7))
    fs = int(rng.integers(0, 4))
    fd = int(rng.integers(max(0, fs - Ld + 1), fs + Ls))          # overlapping layer windows
    lo_min, hi_max = max(fs, fd), min(fs + Ls, fd + Ld)
    lo = int(rng.integers(lo_min, hi_max + 1))
    hi = int(rng.integers(lo, hi_max + 1))
    mode = rng.choice(["two_pools", "same_pool", "swap_out", "swap_in", "heads", "fanout"],
                      p=[0.35, 0.2, 0.1, 0.1, 0.15, 0.1])
    kernel = int(rng.choice([wk.KERNEL_TMA, wk.KERNEL_SIMT, wk.KERNEL_COPY_ENGINE], p=[0.45, 0.4, 0.15]))
    if mode in ("swap_out", "swap_in") and rng.random() < 0.4:
        kernel = wk.KERNEL_STAGED  # staged copy engines: host-side table read on the CPU
    big = rng.random() < 0.2                               # a fifth span many CTAs / windows
    nbs, nbd = (int(rng.integers(1, 2000)), int(rng.integers(1, 2000))) if big else \
        (int(rng.integers(1, 160)), int(rng.integers(1, 160)))
    n = int(rng.integers(0, min(nbs, nbd) + 1)) if rng.random() > 0.05 else 0

    if mode == "same_pool":
        nbd = nbs
        Ld, fd = Ls, fs
        lo, hi = fs, fs + Ls
        perm = rng.permutation(nbs)
        n = min(n, nbs // 2)
        sbt = perm[:n].astype(np.int32)
        free = perm[n:]
        dbt = np.where(rng.random(n) < 0.2, sbt, free[:n]).astype(np.int32)  # identity pairs allowed
    else:
        sbt = rng.integers(0, nbs, n).astype(np.int32)       # duplicates = fan-out (R5)
        dbt = rng.permutation(nbd)[:n].astype(np.int32)
    if mode in ("swap_out", "swap_in"):
        Ld, fd, lo, hi = Ls, fs, fs, fs + Ls

    src_loc = "host" if mode == "swap_in" else "device"
    dst_loc = "host" if mode == "swap_out" else "device"
    path = wk.PATH_HOST if mode in ("swap_out", "swap_in") else wk.PATH_INTRA
    tuning = draw_tuning(rng, kernel)
    wk.set_tuning(path, **tuning)
    # device -> device ops with an SM kernel: sometimes burst-paced or step-released slices
    pace = str(rng.choice(["none", "burst", "stepped"], p=[0.6, 0.2, 0.2])) if mode == "two_pools" else "none"

    Hd = int(rng.integers(1, 7)) if mode == "heads" else H   # TP reshard: head counts differ (R24)
    src, s0 = filled(rng, Ls, H, d, bs, eb, nbs, fs, loc=src_loc)
    if mode == "same_pool":
        dst, d0 = src, s0
    else:
        dst, d0 = filled(rng, Ld, Hd, d, bs, eb, nbd, fd, loc=dst_loc)
    flags0 = [dst.layer_count(l) for l in range(fd, fd + Ld)]
    want = d0.copy()
    ce = kernel in (wk.KERNEL_COPY_ENGINE, wk.KERNEL_STAGED)  # tables read on the CPU
    to = (lambda a: torch.as_tensor(a).pin_memory()) if ce else (lambda a: torch.as_tensor(a, device=DEV))
    ts, td = to(sbt), to(dbt)

    if mode == "fanout":  # one source table object, k destinations in one launch (NEXT-3)
        k = int(rng.integers(2, 6))
        extra = [filled(rng, Ld, H, d, bs, eb, int(rng.integers(n, n + 40)) if n else 1, fd)
                 for _ in range(k - 1)]
        tabs = [dbt] + [rng.permutation(p.desc.n_blocks)[:n].astype(np.int32) for p, _ in extra]
        if kernel in (wk.KERNEL_TMA, wk.KERNEL_SIMT) and n > 0 and hi > lo and rng.random() < 0.3:
            # the batch burst-paced: slices of the shared unit space between pace kernels
            payload = 2 * (hi - lo) * n * (H * bs * d * eb)
            pace = "burst"
            wk.set_tuning(path, **{**tuning, "max_ctas": 0,
                                   "rate_mbps": max(1, int(payload / int(rng.integers(1, 6)) / 2e-3 / 1e6))})
        wk.migrate_batch(src, [(q, ts, to(t), n) for q, t in zip([dst] + [p for p, _ in extra], tabs)], lo, hi)
        for (q, q0), t in zip(extra, tabs[1:]):
            w = q0.copy()
            assert O.migrate(s0, geom(src), sbt, w, geom(q), t, lo, hi) == O.OK
            assert np.array_equal(read(q), w), dict(fan=k, n=n)
        assert O.migrate(s0, geom(src), sbt, want, geom(dst), dbt, lo, hi) == O.OK
    elif mode == "heads":
        sh0 = int(rng.integers(0, H))
        nh = int(rng.integers(1, min(H - sh0, Hd) + 1))
        dh0 = int(rng.integers(0, Hd - nh + 1))
        st = O.migrate_heads(s0, geom(src), sbt, want, geom(dst), dbt, lo, hi, sh0, dh0, nh)
        assert st == O.OK
        wk.migrate_heads(src, ts, dst, td, sh0, dh0, nh, n=n, layer_lo=lo, layer_hi=hi)
    elif mode == "same_pool":
        assert O.compact(want, geom(src), sbt, dbt) == O.OK
        wk.compact(src, ts, td, n=n)
    else:
        assert O.migrate(s0, geom(src), sbt, want, geom(dst), dbt, lo, hi) == O.OK
        if mode == "swap_out":
            wk.swap_out(src, ts, dst, td, n=n)
        elif mode == "swap_in":
            wk.swap_in(src, ts, dst, td, n=n)
        elif kernel in (wk.KERNEL_TMA, wk.KERNEL_SIMT) and pace != "none" and n > 0 and hi > lo:
            payload = 2 * (hi - lo) * n * (H * bs * d * eb)
            k = int(rng.integers(1, 7))  # slices the op is cut into (about)
            if pace == "burst":  # rate-limited, no CTA cap: slices between pace kernels
                rate_mbps = max(1, int(payload / k / 2e-3 / 1e6))  # ~k slices of 2 ms budget
                wk.migrate_ex(src, ts, dst, td, wk.tuning(**{**tuning, "max_ctas": 0, "rate_mbps": rate_mbps}),
                              n=n, layer_lo=lo, layer_hi=hi)
            else:  # stepped: slices released by another stream's step signals
                counter = torch.zeros(1, dtype=torch.int32, device=DEV)
                s_mig, s_dec = torch.cuda.Stream(DEV), torch.cuda.Stream(DEV)
                wk.set_tuning(path, **tuning)
                n0 = wk.launch_count()
                wk.migrate_stepped(src, ts, dst, td, counter, first_step=1, bytes_per_step=-(-payload // k),
                                   n=n, layer_lo=lo, layer_hi=hi, stream=s_mig)
                for _ in range(wk.launch_count() - n0):
                    wk.step_signal(counter, stream=s_dec)
                s_mig.synchronize()
        else:
            wk.migrate(src, ts, dst, td, n=n, layer_lo=lo, layer_hi=hi)
    got = read(dst)
    ctx = dict(mode=str(mode), kernel=kernel, tuning=tuning, L=(Ls, Ld), first=(fs, fd), lo=lo, hi=hi,
               H=(H, Hd), d=d, bs=bs, eb=eb, nb=(nbs, nbd), n=n, pace=pace)
    assert np.array_equal(got, want), ctx
    # flags (R19, R23): an op with n > 0 and lo < hi adds exactly 1 to every dst layer flag;
    # an empty op adds nothing
    bump = 1 if (n > 0 and hi > lo) else 0
    assert [dst.layer_count(l) for l in range(fd, fd + Ld)] == [f + bump for f in flags0], ctx
