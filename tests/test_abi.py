"""CPU-only checks of the C-ABI library: it loads, exports every symbol include/wind_kv.h
declares, and its host-side logic (planners, status strings, tuning) agrees with the
oracle.  No compute calls (there is no GPU here)."""
import os
import re

import numpy as np
import pytest

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk
from paper_conf_isca_fenghzly025_b200 import _build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module", autouse=True)
def built():
    _build.build()
    yield


def header_functions():
    txt = open(os.path.join(ROOT, "include", "wind_kv.h")).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(wind_kv_[a-z_0-9]+)\s*\(", txt)))


def test_header_and_binding_agree():
    assert header_functions() == sorted(wk.EXPORTED_SYMBOLS)


def test_library_exports_every_symbol():
    L = wk.lib()
    for name in header_functions():
        assert hasattr(L, name), name
    # and nothing in the dynamic symbol table is missing from the header
    out = os.popen(f"nm -D --defined-only {wk.LIB_PATH}").read()
    exported = set(re.findall(r"\bT (wind_kv_\w+)", out))
    assert exported == set(header_functions())


def test_status_strings_match_abi_codes():
    L = wk.lib()
    for code, name in wk.STATUS.items():
        assert L.wind_kv_status_string(code).decode() == name
    # the oracle re-declares the same numeric codes independently
    for name in ("OK", "INVALID_ARG", "GEOMETRY", "LAYER_RANGE", "BLOCK_RANGE", "DUP_DST", "ALIAS",
                 "OOM", "UNSUPPORTED"):
        code = getattr(O, name)
        assert wk.STATUS[code].endswith(name)


def test_version_and_launch_count():
    assert "sm_100a" in wk.version()
    assert wk.launch_count() == 0


def test_plan_compact_matches_oracle_exhaustive():
    for mask in range(1 << 10):
        live = np.array([(mask >> b) & 1 for b in range(10)], np.uint8)
        s1, d1 = wk.plan_compact(live)
        s2, d2 = O.plan_compact(live)
        np.testing.assert_array_equal(s1, s2)
        np.testing.assert_array_equal(d1, d2)


def test_plan_compact_large_random():
    rng = np.random.default_rng(3)
    for _ in range(20):
        live = (rng.random(5000) < rng.random()).astype(np.uint8)
        s1, d1 = wk.plan_compact(live)
        s2, d2 = O.plan_compact(live)
        np.testing.assert_array_equal(s1, s2)
        np.testing.assert_array_equal(d1, d2)


def test_plan_rebalance_matches_oracle():
    """The plan's CHOICE follows a reading (R26, a heuristic the paper does not define), but library
    and oracle implement the same stated rule and must agree exactly."""
    from windgen import skewed_placement, lengths_longtail, blocks_for_tokens
    for G in (1, 2, 4, 8):
        for seed in range(6):
            R = 300
            gpu = skewed_placement(R, G, seed)
            blocks = blocks_for_tokens(lengths_longtail(R, seed + 50), 16).astype(np.int32)
            blocks[::17] = 0
            o1, m1 = wk.plan_rebalance(G, gpu, blocks)
            o2, m2 = O.plan_rebalance(G, gpu, blocks)
            np.testing.assert_array_equal(o1, o2)
            assert m1 == m2


def test_tuning_roundtrip_and_bounds():
    old = wk.get_tuning(wk.PATH_PEER)
    wk.set_tuning(wk.PATH_PEER, kernel=wk.KERNEL_TMA, ctas_per_sm=2, stage_bytes=16384, stages=4)
    t = wk.get_tuning(wk.PATH_PEER)
    assert (t["kernel"], t["ctas_per_sm"], t["stage_bytes"], t["stages"]) == (1, 2, 16384, 4)
    with pytest.raises(wk.WindKVError) as e:
        wk.set_tuning(wk.PATH_PEER, stage_bytes=100)
    assert e.value.status == -1
    with pytest.raises(wk.WindKVError):
        wk.set_tuning(wk.PATH_PEER, stage_bytes=131072, stages=4)  # > 227 KiB smem
    with pytest.raises(wk.WindKVError) as e:  # staged copy engines: HOST path only
        wk.set_tuning(wk.PATH_PEER, kernel=wk.KERNEL_STAGED)
    assert e.value.status == -1
    wk.set_tuning(wk.PATH_PEER, **{k: v for k, v in old.items()})
    assert wk.get_tuning(wk.PATH_PEER) == old
    old_h = wk.get_tuning(wk.PATH_HOST)
    wk.set_tuning(wk.PATH_HOST, **{**old_h, "kernel": wk.KERNEL_STAGED})
    assert wk.get_tuning(wk.PATH_HOST)["kernel"] == wk.KERNEL_STAGED
    wk.set_tuning(wk.PATH_HOST, **old_h)
    assert wk.get_tuning(wk.PATH_HOST) == old_h


def test_null_arguments_fail_cleanly_without_gpu():
    L = wk.lib()
    assert L.wind_kv_migrate(None, None, None, None, 0, 0, 0, None) == -1
    assert L.wind_kv_pool_create(None, None, None) == -1
    assert L.wind_kv_pool_destroy(None) == 0
    assert "NULL" in wk.last_error()
    assert L.wind_kv_route(None, None, None, None, None) == -1


def test_binding_accepts_only_int32_device_accessible_tables():
    """The binding marshals block tables as raw int32 addresses the kernels read on the
    device: other dtypes would be reinterpreted, pageable host memory is not accessible."""
    import torch
    with pytest.raises(TypeError):
        wk._ptr(torch.zeros(4, dtype=torch.uint8))
    with pytest.raises(TypeError):
        wk._ptr(torch.zeros(4, dtype=torch.int64))
    with pytest.raises(ValueError):
        wk._ptr(torch.zeros(4, dtype=torch.int32))  # pageable CPU memory
    with pytest.raises(ValueError):
        wk._ptr(torch.zeros(8, dtype=torch.int32)[::2])  # not contiguous
    assert wk._ptr(None) is None and wk._ptr(1234) == 1234


def test_plan_compact_worked_example():
    """The library's planner on the hand-worked O6 examples (tests/golden/)."""
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "o6_compaction_worked_example.json")))
    for c in g["cases"]:
        s, d = wk.plan_compact(np.asarray(c["live"], np.uint8))
        assert s.tolist() == c["src_bt"] and d.tolist() == c["dst_bt"], c


def test_plan_rebalance_worked_examples():
    """The library's rebalance planner on the hand-worked R26 examples (tests/golden/)."""
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "r26_rebalance_worked_examples.json")))
    for c in g["cases"]:
        out, n = wk.plan_rebalance(c["n_gpus"], c["req_gpu"], c["req_blocks"])
        assert out.tolist() == c["out_gpu"] and n == c["n_moves"], c
