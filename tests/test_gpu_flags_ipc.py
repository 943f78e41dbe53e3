"""GPU: layer-completion flags (A5), cross-process pools (CUDA IPC, the
prefill->decode hand-off mechanics, A4), full-size parity at the bench configuration, and
the device-side input generator against its host twin."""
import math
import multiprocessing as mp
import os
import sys

import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
import windgen
import windgen.cuda as wg
from windgen import KVShape, SHAPES, migration_case, content_bytes

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def geom(p: wk.Pool) -> O.Geom:
    d = p.desc
    return O.Geom(d.first_layer, d.n_layers, d.n_kv_heads, d.head_dim, d.block_size, d.elem_bytes,
                  d.n_blocks)


def pattern_pool(sh, nb, seed, tag, loc="device"):
    p = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nb, loc=loc)
    if loc == "device":
        wg.fill(p.base, p.nbytes, 0, seed, tag)
    else:
        p.tensor().copy_(torch.from_numpy(content_bytes(seed, tag, 0, p.nbytes)))
    return p


@pytest.fixture(autouse=True)
def default_tuning():
    saved = {p: wk.get_tuning(p) for p in (wk.PATH_INTRA, wk.PATH_PEER, wk.PATH_HOST)}
    yield
    for p, t in saved.items():
        wk.set_tuning(p, **t)


def test_device_generator_matches_host_generator():
    buf = torch.empty(1 << 20, dtype=torch.uint8, device=DEV)
    for off in (0, 8, 4096 * 1000 + 8):
        wg.fill(buf.data_ptr(), buf.numel(), off, 3002, 5)
        torch.cuda.synchronize()
        np.testing.assert_array_equal(buf.cpu().numpy(), content_bytes(3002, 5, off, buf.numel()))
    key = windgen.content_key(3002, 5)
    cnt, first = wg.check_chunks(buf.data_ptr(), 4096, [0, 4096], [off, off + 4096], [key, key])
    assert cnt == 0
    cnt, first = wg.check_chunks(buf.data_ptr(), 4096, [0, 4096], [off, off], [key, key])
    assert cnt == 1 and first == 1


@pytest.mark.parametrize("kernel", [wk.KERNEL_TMA, wk.KERNEL_SIMT])
@pytest.mark.parametrize("n", [192, 16])
def test_layer_flags_ordering_property(kernel, n):
    """P8: a consumer stream that waits on layer_done[l] >= ticket and then snapshots layer
    l's destination chunks always sees the migrated bytes (never the old ones), trial after
    trial, for every layer.  n = 192: more work units per plane than CTAs (grid-stride
    dealing, layers complete while the op runs); n = 16: fewer (contiguous per-CTA ranges)."""
    wk.set_tuning(wk.PATH_INTRA, kernel=kernel)
    sh = KVShape("opt13b-8L", 8, 40, 128, 2)  # C = 160 KiB, 1.25 MiB per block-layer pair
    nb = 220
    rng = np.random.default_rng(0)
    sbt = rng.permutation(nb)[:n].astype(np.int32)
    dbt = rng.permutation(nb)[:n].astype(np.int32)
    src = pattern_pool(sh, nb, 77, 1)
    dst = pattern_pool(sh, nb, 77, 2)
    C = sh.chunk_bytes
    sample = np.sort(rng.choice(n, min(12, n), replace=False))
    view = dst.tensor().view(sh.n_layers, 2, nb, C)
    want = src.tensor().view(sh.n_layers, 2, nb, C)[:, :, torch.as_tensor(sbt[sample], device=DEV)].clone()
    didx = torch.as_tensor(dbt[sample].astype(np.int64), device=DEV)
    ts, td = torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV)
    mover = torch.cuda.Stream(DEV)
    consumer = torch.cuda.Stream(DEV)
    trials = 1000
    bad = torch.zeros((), dtype=torch.int64, device=DEV)
    snap = torch.empty((2, len(sample), C), dtype=torch.uint8, device=DEV)
    for k in range(trials):
        with torch.cuda.stream(mover):
            wg.fill(dst.base, dst.nbytes, 0, 77, 2, mover.cuda_stream)  # reset to old bytes
        wk.migrate(src, ts, dst, td, stream=mover)
        t = dst.layer_ticket()
        for l in range(sh.n_layers):
            wk.layer_wait(dst, l, t, stream=consumer)
            with torch.cuda.stream(consumer):
                snap.copy_(view[l][:, didx])
                bad += (snap != want[l]).any().to(torch.int64)
        mover.wait_stream(consumer)  # next trial's reset only after the snapshots
    torch.cuda.synchronize()
    assert bad.item() == 0
    assert all(dst.layer_count(l) == trials for l in range(sh.n_layers))


def test_layer_flags_host_pool_swap_out():
    """Swap-out flags live in mapped host memory: once the host sees layer_done[l] >=
    ticket, that layer's host bytes are final."""
    case = migration_case("C1", scale=0.5)
    sh = case.shape
    dev = pattern_pool(sh, case.nb_src, 5, 1)
    host = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, case.n,
                   loc="host")
    hbt = torch.arange(case.n, dtype=torch.int32, device=DEV)
    ht = host.tensor().view(sh.n_layers, 2, case.n, -1)
    want = torch.from_numpy(content_bytes(5, 1, 0, dev.nbytes)).view(sh.n_layers, 2, case.nb_src, -1)
    want = want[:, :, torch.as_tensor(case.src_bt.astype(np.int64))]
    tsrc = torch.as_tensor(case.src_bt, device=DEV)
    rng = np.random.default_rng(0)
    for trial in range(1, 301):
        pick = torch.as_tensor(rng.choice(case.n, 3, replace=False).astype(np.int64))
        ht[:, :, pick] = 0  # stale bytes the check would see if a flag ran ahead of its data
        wk.swap_out(dev, tsrc, host, hbt)
        for l in range(sh.n_layers):
            while host.layer_count(l) < trial:
                pass
            assert torch.equal(ht[l][:, pick], want[l][:, pick]), (trial, l)
        torch.cuda.synchronize()
    assert torch.equal(ht, want)


# ---------------------------------------------------------------------- IPC (A4)

def _owner(q_out, q_in, shape_args, nb, seed, tag):
    sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
    import torch  # noqa
    import paper_conf_isca_fenghzly025_b200 as wk2
    import windgen.cuda as wg2
    p = wk2.Pool(*shape_args, nb)
    wg2.fill(p.base, p.nbytes, 0, seed, tag)
    torch.cuda.synchronize()
    q_out.put(p.export())
    msg = q_in.get(timeout=300)  # wait for the peer's migration
    torch.cuda.synchronize()
    q_out.put((p.tensor().cpu().numpy(), [p.layer_count(l) for l in range(shape_args[0])], msg))
    q_in.get(timeout=300)


def test_ipc_push_and_pull_between_processes():
    """The decode process owns and exports its pool; the prefill process imports it and
    pushes blocks into it (and pulls some back) — CUDA IPC + layer flags across processes.
    One GPU here, so both map the same device; the code path is the multi-GPU one."""
    sh = KVShape("t", 4, 8, 128, 2)
    shape_args = (sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes)
    ctx = mp.get_context("spawn")
    q_out, q_in = ctx.Queue(), ctx.Queue()
    proc = ctx.Process(target=_owner, args=(q_out, q_in, shape_args, 90, 9, 2))
    proc.start()
    try:
        handle = q_out.get(timeout=300)
        remote = wk.Pool.import_(handle, 0)
        assert remote.desc.n_blocks == 90 and remote.nbytes == sh.n_layers * 2 * 90 * sh.chunk_bytes
        src = pattern_pool(sh, 120, 9, 1)
        # same GPU: INTRA route, unless WIND_KV_FORCE_PEER_ROUTE=1 (test_gpu_sys_scope.py) makes
        # ops with an imported pool take the PEER route (PEER tuning, system-scope flags)
        forced = os.environ.get("WIND_KV_FORCE_PEER_ROUTE") == "1"
        want_path = wk.PATH_PEER if forced else wk.PATH_INTRA
        assert wk.route(src, remote) == (0, want_path, forced)
        assert wk.route(remote, src) == (0, want_path, forced)
        rng = np.random.default_rng(4)
        sbt = rng.permutation(120)[:50].astype(np.int32)
        dbt = rng.permutation(90)[:50].astype(np.int32)
        s = torch.cuda.Stream(DEV)
        # one batched launch pushes into the imported pool AND a local pool (A8 sender side)
        side = pattern_pool(sh, 70, 9, 4)
        sb2 = rng.permutation(120)[:40].astype(np.int32)
        db2 = rng.permutation(70)[:40].astype(np.int32)
        # tables are borrowed until the ops on `s` complete: keep them referenced
        tabs = [torch.as_tensor(x, device=DEV) for x in (sbt, dbt, sb2, db2, dbt[:10])]
        wk.migrate_batch(src, [(remote, tabs[0], tabs[1]), (side, tabs[2], tabs[3])], 1, 4, stream=s)
        t = remote.layer_ticket()
        for l in range(4):
            wk.layer_wait(remote, l, t, stream=s)
        flags_h = torch.zeros(4, dtype=torch.int32).pin_memory()
        remote.read_flags(flags_h, stream=s)  # async read of the peer's flags
        # pull: remote -> a local pool
        back = pattern_pool(sh, 60, 9, 3)
        pb = np.arange(10, dtype=np.int32)
        tabs.append(torch.as_tensor(pb, device=DEV))
        wk.migrate(remote, tabs[4], back, tabs[5], stream=s)
        s.synchronize()
        q_in.put("done")
        got, counts, _ = q_out.get(timeout=300)
        # oracle: the owner's pool after the push
        g_src = geom(src)
        g_rem = O.Geom(0, 4, 8, 128, 16, 2, 90)
        want = content_bytes(9, 2, 0, got.size)
        assert O.migrate(content_bytes(9, 1, 0, src.nbytes), g_src, sbt, want, g_rem, dbt, 1, 4) == O.OK
        np.testing.assert_array_equal(got, want)
        assert counts == [1, 1, 1, 1] and flags_h.tolist() == [1, 1, 1, 1]
        want_side = content_bytes(9, 4, 0, side.nbytes)
        assert O.migrate(content_bytes(9, 1, 0, src.nbytes), g_src, sb2, want_side, geom(side), db2,
                         1, 4) == O.OK
        np.testing.assert_array_equal(side.tensor().cpu().numpy(), want_side)
        want_b = content_bytes(9, 3, 0, back.nbytes)
        assert O.migrate(want, g_rem, dbt[:10], want_b, geom(back), pb, 0, 4) == O.OK
        torch.cuda.synchronize()
        np.testing.assert_array_equal(back.tensor().cpu().numpy(), want_b)
        remote.destroy()
        q_in.put("bye")
    finally:
        proc.join(timeout=120)
        if proc.is_alive():
            proc.kill()
    assert proc.exitcode == 0


def test_import_in_same_process_is_unsupported():
    sh = KVShape("t", 1, 2, 64, 2)
    p = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, 4)
    with pytest.raises(wk.WindKVError) as e:
        wk.Pool.import_(p.export(), 0)
    assert e.value.status == -10


# ------------------------------------------------------------ full-size (bench config)

@pytest.mark.parametrize("variant", ["shuffled", "sequential"])
def test_full_size_c2_parity_every_chunk(variant):
    """BJ:configs[1] at full size (35 GiB payload, ~100 GiB of pools) in the launch
    configuration bench.py times: EVERY destination chunk is checked on the device against
    the oracle's P2 closed form (origin offset per chunk), plus a sampled host-side
    byte comparison against the numpy generator."""
    case = migration_case("C2", variant=variant)
    sh = case.shape
    src = pattern_pool(sh, case.nb_src, case.content_seed, case.src_tag)
    dst = pattern_pool(sh, case.nb_dst, case.content_seed, case.dst_tag)
    s = torch.cuda.Stream(DEV)
    ts, td = torch.as_tensor(case.src_bt, device=DEV), torch.as_tensor(case.dst_bt, device=DEV)
    wk.migrate(src, ts, dst, td, stream=s)  # tables borrowed until the op completes
    s.synchronize()
    gs, gd = geom(src), geom(dst)
    from_src, off = O.expected_origin(gs, case.src_bt, gd, case.dst_bt, 0, sh.n_layers)
    C = sh.chunk_bytes
    ks, kd = windgen.content_key(case.content_seed, case.src_tag), windgen.content_key(case.content_seed, case.dst_tag)
    keys = np.where(from_src == 1, np.uint64(ks), np.uint64(kd))
    dst_off = np.arange(from_src.size, dtype=np.int64) * C
    cnt, first = wg.check_chunks(dst.base, C, dst_off, off, keys)
    assert cnt == 0, f"{cnt} chunks differ, first {first}"
    assert int(from_src.sum()) == 2 * sh.n_layers * case.n
    rng = np.random.default_rng(1)
    t = dst.tensor()
    for c in rng.choice(from_src.size, 24, replace=False).tolist():
        want = content_bytes(case.content_seed, case.src_tag if from_src[c] else case.dst_tag, int(off[c]), C)
        np.testing.assert_array_equal(t[c * C:(c + 1) * C].cpu().numpy(), want)
