"""Run one bench scenario alone on cuda:0 (development helper): python scripts/run_scenario.py <name>"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402

name = sys.argv[1]
peaks = bench.load_peaks()
T, S = wk.KERNEL_TMA, wk.KERNEL_SIMT
small_footprint = [
    ("tma48kx4_cap4", dict(kernel=T, stage_bytes=49152, stages=4, store_lag=2, ctas_per_sm=1, max_ctas=4)),
    ("tma16kx4_cap8", dict(kernel=T, stage_bytes=16384, stages=4, store_lag=2, ctas_per_sm=1, max_ctas=8)),
    ("tma16kx4_cap16", dict(kernel=T, stage_bytes=16384, stages=4, store_lag=2, ctas_per_sm=1, max_ctas=16)),
    ("tma8kx4_cap16", dict(kernel=T, stage_bytes=8192, stages=4, store_lag=2, ctas_per_sm=1, max_ctas=16)),
    ("simt32k_cap4", dict(kernel=S, stage_bytes=32768, stages=6, ctas_per_sm=1, max_ctas=4)),
    ("simt32k_cap8", dict(kernel=S, stage_bytes=32768, stages=6, ctas_per_sm=1, max_ctas=8)),
    ("tma48kx4_cap4_ef", dict(kernel=T, stage_bytes=49152, stages=4, store_lag=2, ctas_per_sm=1, max_ctas=4,
                              evict_first=True)),
    ("tma48kx4_cap2", dict(kernel=T, stage_bytes=49152, stages=4, store_lag=2, ctas_per_sm=1, max_ctas=2)),
    ("tma16kx3_cap2", dict(kernel=T, stage_bytes=16384, stages=3, store_lag=1, ctas_per_sm=1, max_ctas=2)),
    ("tma16kx3_rate50", dict(kernel=T, stage_bytes=16384, stages=3, store_lag=1, ctas_per_sm=1, max_ctas=0,
                             rate_mbps=50000)),
    ("simt32k_rate50", dict(kernel=S, stage_bytes=32768, stages=4, ctas_per_sm=1, max_ctas=2, rate_mbps=50000)),
    ("ce_rate50", dict(kernel=3, stage_bytes=49152, stages=4, rate_mbps=50000)),
]
fn = {"interference": lambda: bench.run_interference(wk, 0, peaks),
      "interference_configs": lambda: bench.run_interference(wk, 0, peaks, n_victim_steps=30,
                                                             configs=small_footprint),
      "pressure": lambda: bench.run_pressure(wk, 0),
      "c1_intra": lambda: bench.run_c1_intra(wk, 0, peaks),
      "interference_rw": lambda: bench.run_interference(wk, 0, peaks, n_victim_steps=40, configs=[
          (n, c) for n, c in [
              ("control_no_migration", {**wk.get_tuning(wk.PATH_INTRA), "null_feeder": True}),
              ("rate50GBs", {**wk.get_tuning(wk.PATH_INTRA), "rate_mbps": 50000}),
              ("rate50GBs_evict_first", {**wk.get_tuning(wk.PATH_INTRA), "rate_mbps": 50000, "evict_first": 1}),
              ("copy_engines_rate50GBs", {**wk.get_tuning(wk.PATH_INTRA), "kernel": 3, "rate_mbps": 50000}),
              ("hbm_reads_only_swap_out_sm8", {"op": "swap_out", **wk.get_tuning(wk.PATH_HOST), "kernel": 1}),
              ("hbm_writes_only_swap_in_sm8", {"op": "swap_in", **wk.get_tuning(wk.PATH_HOST), "kernel": 1}),
              ("swap_out_staged_ce", {"op": "swap_out", **wk.get_tuning(wk.PATH_HOST), "kernel": 4}),
              ("swap_in_staged_ce", {"op": "swap_in", **wk.get_tuning(wk.PATH_HOST), "kernel": 4}),
              ("hbm_reads_only_swap_out_sm8_b", {"op": "swap_out", **wk.get_tuning(wk.PATH_HOST), "kernel": 1}),
              ("hbm_writes_only_swap_in_sm8_b", {"op": "swap_in", **wk.get_tuning(wk.PATH_HOST), "kernel": 1}),
          ]]),
      "interference_swap": lambda: bench.run_interference(wk, 0, peaks, n_victim_steps=40, configs=[
          (n, {"op": op, **wk.get_tuning(wk.PATH_HOST), **c}) for n, op, c in [
              ("staged_out_default", "swap_out", dict(kernel=4)),
              ("staged_in_default", "swap_in", dict(kernel=4)),
              ("staged_out_hidden2", "swap_out", dict(kernel=4, max_ctas=2)),
              ("staged_out_hidden32", "swap_out", dict(kernel=4, max_ctas=32)),
              ("sm_out_tma8", "swap_out", dict(kernel=1)),
              ("sm_out_tma8_rate45", "swap_out", dict(kernel=1, rate_mbps=45000)),
              ("sm_out_tma8_rate30", "swap_out", dict(kernel=1, rate_mbps=30000)),
              ("sm_out_tma2", "swap_out", dict(kernel=1, max_ctas=2)),
              ("sm_out_tma1", "swap_out", dict(kernel=1, max_ctas=1)),
              ("sm_out_simt8", "swap_out", dict(kernel=2, max_ctas=8, stage_bytes=32768)),
              ("sm_out_simt2", "swap_out", dict(kernel=2, max_ctas=2, stage_bytes=32768)),
              ("sm_in_tma8", "swap_in", dict(kernel=1)),
          ]]),
      "interference_swap2": lambda: bench.run_interference(wk, 0, peaks, n_victim_steps=40, configs=[
          (n, {"op": op, **wk.get_tuning(wk.PATH_HOST), **c}) for n, op, c in [
              ("staged_out_h4", "swap_out", dict(kernel=4, max_ctas=4)),
              ("staged_in_h4", "swap_in", dict(kernel=4, max_ctas=4)),
              ("staged_out_h2", "swap_out", dict(kernel=4, max_ctas=2)),
              ("staged_in_h2", "swap_in", dict(kernel=4, max_ctas=2)),
              ("sm_out_tma2", "swap_out", dict(kernel=1, max_ctas=2)),
              ("sm_out_tma3", "swap_out", dict(kernel=1, max_ctas=3)),
              ("sm_out_tma4", "swap_out", dict(kernel=1, max_ctas=4)),
              ("sm_out_tma8_rate50", "swap_out", dict(kernel=1, max_ctas=8, rate_mbps=50000)),
              ("sm_in_tma2", "swap_in", dict(kernel=1, max_ctas=2)),
              ("sm_in_tma4", "swap_in", dict(kernel=1, max_ctas=4)),
              ("sm_in_tma8", "swap_in", dict(kernel=1, max_ctas=8)),
              ("staged_out_h4_b", "swap_out", dict(kernel=4, max_ctas=4)),
              ("sm_out_tma2_b", "swap_out", dict(kernel=1, max_ctas=2)),
          ]]),
      "interference_ce": lambda: bench.run_interference(wk, 0, peaks, n_victim_steps=40, configs=[
          (n, {**wk.get_tuning(wk.PATH_INTRA), **c}) for n, c in [
              ("ce_rate50", dict(kernel=3, rate_mbps=50000)),
              ("ce_rate150", dict(kernel=3, rate_mbps=150000)),
              ("ce_rate300", dict(kernel=3, rate_mbps=300000)),
              ("ce_rate450", dict(kernel=3, rate_mbps=450000)),
              ("ce_rate600", dict(kernel=3, rate_mbps=600000)),
              ("ce_unlimited", dict(kernel=3, rate_mbps=0)),
              ("ce_rate300_b", dict(kernel=3, rate_mbps=300000)),
              ("ce_rate150_b", dict(kernel=3, rate_mbps=150000))]]),
      "policy": lambda: bench.run_policy_profile(wk, 0),
      "stall_free": lambda: bench.run_stall_free(wk, 0),
      "handoff": lambda: bench.run_handoff(wk, 0),
      "next3": lambda: bench.run_next3(wk, 0, peaks),
      "partition": lambda: bench.run_interference(wk, 0, peaks, n_victim_steps=30, configs=[
          (n, {**wk.get_tuning(wk.PATH_INTRA), **c}) for n, c in [
              ("cap8", dict(max_ctas=8)), ("rate50GBs", dict(rate_mbps=50000)),
              ("partition8_tma", dict(partition=8)), ("partition8_tma_rate50GBs", dict(partition=8, rate_mbps=50000)),
              ("partition8_tma_rate150GBs", dict(partition=8, rate_mbps=150000)),
              ("copy_engines_rate50GBs", dict(kernel=3, rate_mbps=50000))]])}[name]
print(json.dumps(fn()))
