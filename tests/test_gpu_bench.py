"""GPU: the bench contract end to end (small config), at N = 1 and at N = 2 / 3 under
torchrun with every rank on cuda:0 (WIND_BENCH_ONE_DEVICE: the N > 1 code path — IPC
handle exchange over gloo, pushes into imported pools, batched all-to-all — on one GPU)."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _json_line(out: str) -> dict:
    lines = [l for l in out.splitlines() if l.startswith("{")]
    assert lines, out[-3000:]
    return json.loads(lines[-1])


def test_bench_n1_contract():
    out = subprocess.run([sys.executable, "bench.py", "--steps", "3", "--warmup", "3", "--config", "C1",
                          "--no-scenarios"], cwd=ROOT, capture_output=True, text=True, timeout=600)
    assert out.returncode == 0, out.stderr[-3000:]
    d = _json_line(out.stdout)
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
              "scaling", "vs_baseline", "dtype", "data", "config", "e2e", "gpu_launches", "clocks",
              "roofline", "cpu_baseline"):
        assert k in d, k
    assert d["gpu_launches"] == 3 and d["value"] > 0 and d["roofline"]["bound"] == "hbm"
    assert d["cpu_baseline"]["parity_check_of_this_run"]["ok"] is True
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1


@pytest.mark.parametrize("world", [2, 3])
def test_bench_multirank_on_one_gpu(world):
    env = dict(os.environ, WIND_BENCH_ONE_DEVICE="1")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", str(world),
           "--steps", "3", "--warmup", "3", "--config", "C1", "--a2a-scale", "0.0625"]
    if world > 2:  # every rank's ~40 GB decode-step victim on ONE GPU: only at N = 2 here
        cmd.append("--no-peer-interference")
    out = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900, env=env)
    assert out.returncode == 0, (out.stdout[-2000:], out.stderr[-3000:])
    d = _json_line(out.stdout)
    # launches summed over ranks: one per step per mover (pairs + an unpaired last rank)
    assert d["n_gpus"] == world and d["value"] > 0 and d["gpu_launches"] == 3 * (world // 2 + world % 2)
    assert d["peer_autotune"].get("chosen", "").split("_")[0] in ("push", "pull"), d["peer_autotune"]
    a2a = d["scenarios"]["c5_all_to_all"]
    assert a2a["shuffle"]["blocks_moved"] > 0 and a2a["rebalance"]["aggregate_gbs"] >= 0
    assert "error" not in d["scenarios"], d["scenarios"].get("error")
    pi = d["scenarios"]["c3_peer_interference"]
    if world == 2:  # one pair: both sides measured for every configuration
        for k in ("trickle150GBs", "uncapped", "stepped_avg150GBs", "stepped_avg400GBs"):
            assert pi[k]["source_slowdown"] is not None and pi[k]["destination_slowdown"] is not None, pi
    else:
        assert pi is None
