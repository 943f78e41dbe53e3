"""The peer (NVLink) publication path and peer route on one GPU.  A peer destination's layer flags are
published at SYSTEM scope (fence.acq_rel.sys, red.relaxed.sys on device-memory flags:
wind_kv_kernels.cu arrive_layer / bump_flag) — code that only a cross-device op selects,
and no gpurun call so far had two GPUs.  WIND_KV_FORCE_SYS_SCOPE=1 makes every op publish
that way, so the flag-ordering property test, the layer-streamed prefill hand-off, the
one-launch all-to-all, whole-pool parity and the 400-case random fuzz run here through the
system-scope code with the data on one device.  Run in a subprocess: the variable is read once per process."""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

NODES = [
    "tests/test_gpu_flags_ipc.py::test_layer_flags_ordering_property",
    "tests/test_gpu_handoff.py::test_prefill_overlapped_handoff_matches_oracle",
    "tests/test_gpu_multidevice.py::test_all_to_all_one_launch_per_device",
    "tests/test_gpu_parity.py::test_migrate_c1_all_kernels",
    "tests/test_gpu_parity.py::test_run_coalescing_across_warp_windows",
    "tests/test_gpu_heads.py",
    "tests/test_gpu_fuzz.py",  # 400 random ops (geometry, tables, windows, kernels, swaps)
    "tests/test_gpu_misc.py::test_burst_paced_op_flags_and_parity",
    "tests/test_gpu_misc.py::test_migrate_stepped_releases_slices_per_step",
]


def test_system_scope_publication_path():
    env = dict(os.environ, WIND_KV_FORCE_SYS_SCOPE="1")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-p", "no:cacheprovider",
                        *NODES], cwd=ROOT, env=env, capture_output=True, text=True, timeout=1200)
    tail = (r.stdout + r.stderr)[-3000:]
    assert r.returncode == 0, tail
    assert " passed" in r.stdout, tail


def test_forced_scope_is_reported_by_route():
    code = ("import torch, paper_conf_isca_fenghzly025_b200 as wk\n"
            "a = wk.Pool(2, 2, 64, 16, 2, 4); b = wk.Pool(2, 2, 64, 16, 2, 4)\n"
            "e, p, s = wk.route(a, b)\n"
            "assert (e, p, s) == (0, wk.PATH_INTRA, True), (e, p, s)\n"
            "print('ok')\n")
    env = dict(os.environ, WIND_KV_FORCE_SYS_SCOPE="1")
    r = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=env, capture_output=True, text=True,
                       timeout=300)
    assert r.returncode == 0 and "ok" in r.stdout, (r.stdout + r.stderr)[-2000:]


def test_forced_peer_route_between_processes():
    """WIND_KV_FORCE_PEER_ROUTE=1: ops between this process's pool and a pool imported from
    another process on the same GPU take the PEER route (the PEER tuning — SIMT by default —
    and system-scope publication): the cross-process push / pull / batched push test and the
    N = 2 bench path run through it, byte-exact against the oracle."""
    env = dict(os.environ, WIND_KV_FORCE_PEER_ROUTE="1")
    r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-p", "no:cacheprovider",
                        "tests/test_gpu_flags_ipc.py::test_ipc_push_and_pull_between_processes",
                        "tests/test_gpu_bench.py::test_bench_multirank_on_one_gpu"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=1500)
    tail = (r.stdout + r.stderr)[-3000:]
    assert r.returncode == 0, tail
    assert " passed" in r.stdout, tail
