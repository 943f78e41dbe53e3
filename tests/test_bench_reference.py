"""CPU: bench.py's reference arm (the oracle on the host cores, `--impl reference`) keeps the
bench contract — one JSON line with the wind_kv arm's metric, unit, direction and
config.workload, a cpu_baseline describing the run, and an e2e object — and the argument
checks (W >= 3).  No GPU involved."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run(*args):
    return subprocess.run([sys.executable, "bench.py", *args], cwd=ROOT, capture_output=True, text=True,
                          timeout=300)


def test_reference_arm_contract():
    r = run("--impl", "reference", "--steps", "2", "--warmup", "3", "--config", "C1")
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["unit"] == "GB/s" and d["higher_is_better"] is True
    assert d["metric"].startswith("KV migration GB/s") and d["value"] > 0
    assert d["config"]["workload"].startswith("C1 OPT-125M KV: 256 blocks of 8 requests")
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == d["value"] and cb["sample"]
    assert d["e2e"] == {"value": d["value"], "unit": "GB/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}
    assert d["steps"] == 2 and d["warmup"] == 3


def test_rank_other_than_zero_prints_nothing():
    env = dict(os.environ, RANK="1", WORLD_SIZE="2")
    r = subprocess.run([sys.executable, "bench.py", "--impl", "reference", "--gpus", "2", "--steps", "1",
                        "--warmup", "3", "--config", "C1"], cwd=ROOT, capture_output=True, text=True,
                       timeout=300, env=env)
    assert r.returncode == 0 and not [l for l in r.stdout.splitlines() if l.startswith("{")]


def test_warmup_below_three_is_rejected():
    r = run("--impl", "reference", "--steps", "1", "--warmup", "2")
    assert r.returncode != 0
