"""Full-size parity for every BJ:configs workload, in the launch configuration bench.py
times (default tuning): EVERY destination chunk is checked on the device against the
oracle's P2 closed form (the origin of each chunk), using the windgen device checker.
(C2 is in test_gpu_flags_ipc.py.)"""
import math

import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
import windgen
import windgen.cuda as wg
from windgen import (SHAPES, migration_case, request_lengths, skewed_placement, blocks_for_tokens,
                     live_mask_after_free)

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def geom(p):
    d = p.desc
    return O.Geom(d.first_layer, d.n_layers, d.n_kv_heads, d.head_dim, d.block_size, d.elem_bytes,
                  d.n_blocks)


def pattern_pool(sh, nb, seed, tag):
    p = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nb)
    wg.fill(p.base, p.nbytes, 0, seed, tag)
    return p


def check_all_chunks(dst, from_src, off, C, key_src, key_dst):
    keys = np.where(from_src == 1, np.uint64(key_src), np.uint64(key_dst))
    dst_off = np.arange(from_src.size, dtype=np.int64) * C
    cnt, first = wg.check_chunks(dst.base, C, dst_off, off, keys)
    assert cnt == 0, f"{cnt} chunks differ, first {first}"


@pytest.mark.parametrize("cfg", ["C1", "C3", "C4"])
def test_full_size_migrate(cfg):
    torch.cuda.empty_cache()
    case = migration_case(cfg)
    sh = case.shape
    src = pattern_pool(sh, case.nb_src, case.content_seed, case.src_tag)
    dst = pattern_pool(sh, case.nb_dst, case.content_seed, case.dst_tag)
    wk.migrate(src, torch.as_tensor(case.src_bt, device=DEV), dst, torch.as_tensor(case.dst_bt, device=DEV))
    torch.cuda.synchronize()
    from_src, off = O.expected_origin(geom(src), case.src_bt, geom(dst), case.dst_bt, 0, sh.n_layers)
    assert int(from_src.sum()) == 2 * sh.n_layers * case.n
    check_all_chunks(dst, from_src, off, sh.chunk_bytes,
                     windgen.content_key(case.content_seed, case.src_tag),
                     windgen.content_key(case.content_seed, case.dst_tag))
    assert all(dst.layer_count(l) == 1 for l in range(sh.n_layers))


def test_full_size_c5_compaction():
    """C5 (Llama-3-8B GQA fp8): GPU 0's share of the skewed placement, half the requests
    freed, compacted in place (same pool: snapshot semantics, P2 via the oracle)."""
    torch.cuda.empty_cache()
    sh = SHAPES["C5"]
    lens = request_lengths("C5")
    place = skewed_placement(lens.size, 8, 4005)
    reqb = blocks_for_tokens(lens[place == 0], 16)
    nb = math.ceil(int(reqb.sum()) * 1.1)
    live, _ = live_mask_after_free(nb, reqb, 0.5, 4006)
    sbt, dbt = wk.plan_compact(live)
    pool = pattern_pool(sh, nb, 3005, 7)
    wk.compact(pool, torch.as_tensor(sbt, device=DEV), torch.as_tensor(dbt, device=DEV))
    torch.cuda.synchronize()
    g = geom(pool)
    from_src, off = O.expected_origin(g, sbt, g, dbt, 0, sh.n_layers)
    key = windgen.content_key(3005, 7)
    check_all_chunks(pool, from_src, off, sh.chunk_bytes, key, key)


@pytest.mark.parametrize("pace", ["stepped", "burst"])
def test_full_size_c3_paced(pace):
    """C3 (OPT-66B, 18 GiB) at full size as the round-2 paced forms: wind_kv_migrate_stepped
    (slices of 2 GiB released by another stream's step signals) and a burst-paced rate
    limit (2 TB/s: 4 GB slices, ~5 between pace kernels) — every destination chunk vs the
    oracle's P2 closed form, every layer flag exactly once."""
    torch.cuda.empty_cache()
    case = migration_case("C3")
    sh = case.shape
    src = pattern_pool(sh, case.nb_src, case.content_seed, case.src_tag)
    dst = pattern_pool(sh, case.nb_dst, case.content_seed, case.dst_tag)
    ts, td = torch.as_tensor(case.src_bt, device=DEV), torch.as_tensor(case.dst_bt, device=DEV)
    s = torch.cuda.Stream(DEV)
    n0 = wk.launch_count()
    if pace == "stepped":
        counter = torch.zeros(1, dtype=torch.int32, device=DEV)
        wk.migrate_stepped(src, ts, dst, td, counter, first_step=1, bytes_per_step=2 << 30, stream=s)
        slices = wk.launch_count() - n0
        assert 8 <= slices <= 10  # 18 GiB / 2 GiB
        sig = torch.cuda.Stream(DEV)
        for _ in range(slices):
            wk.step_signal(counter, stream=sig)
    else:
        wk.migrate_ex(src, ts, dst, td, wk.tuning(rate_mbps=2_000_000, max_ctas=0), stream=s)
        assert 9 <= wk.launch_count() - n0 <= 13  # 1 + 2 x ~5 slices of 4 GB
    torch.cuda.synchronize()
    from_src, off = O.expected_origin(geom(src), case.src_bt, geom(dst), case.dst_bt, 0, sh.n_layers)
    check_all_chunks(dst, from_src, off, sh.chunk_bytes,
                     windgen.content_key(case.content_seed, case.src_tag),
                     windgen.content_key(case.content_seed, case.dst_tag))
    assert all(dst.layer_count(l) == 1 for l in range(sh.n_layers))
