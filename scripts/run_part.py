"""Development helper: one bench.py scenario alone, printed as one JSON line.
usage: python scripts/run_part.py c1_intra|interference|decode_step|pacer_footprint|burst_period|burst_grid|burst|proxy|handoff|stall_free|pressure|next3|policy"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402

peaks = bench.load_peaks()
name = sys.argv[1]
fn = {"c1_intra": lambda: bench.run_c1_intra(wk, 0, peaks),
      "interference": lambda: bench.run_interference(wk, 0, peaks),
      "decode_step": lambda: bench.run_interference(wk, 0, peaks, victim_kind="decode_step"),
      "burst_grid": lambda: {v: bench.run_interference(wk, 0, peaks, victim_kind=v, configs=[
          (f"rate{r}GBs", {**wk.get_tuning(wk.PATH_INTRA), "max_ctas": 0, "rate_mbps": r * 1000})
          for r in (50, 150)]) for v in ("attention", "decode_step")},
      "burst_period": lambda: bench.run_interference(wk, 0, peaks, victim_kind="decode_step", configs=[
          (f"rate{r}GBs", {**wk.get_tuning(wk.PATH_INTRA), "max_ctas": 0, "rate_mbps": r * 1000})
          for r in (50, 150, 300)]),
      # rate-limited kernels with a smaller on-SM footprint, next to the decode-step victim
      "pacer_footprint": lambda: bench.run_interference(wk, 0, peaks, victim_kind="decode_step", configs=[
          (name, {**wk.get_tuning(wk.PATH_INTRA), "max_ctas": 0, "rate_mbps": 150000, **kw})
          for name, kw in (("rate150_tma_48kx4", {}),
                           ("rate150_tma_16kx4", {"stage_bytes": 16384, "stages": 4, "store_lag": 2}),
                           ("rate150_tma_8kx4", {"stage_bytes": 8192, "stages": 4, "store_lag": 2}),
                           ("rate150_simt", {"kernel": wk.KERNEL_SIMT, "stage_bytes": 32768}),
                           ("rate50_simt", {"kernel": wk.KERNEL_SIMT, "stage_bytes": 32768,
                                            "rate_mbps": 50000}))]),
      # trickle rows only (then the burst rows, which run_interference always adds)
      "burst": lambda: bench.run_interference(wk, 0, peaks, configs=[
          (f"rate{r}GBs", {**wk.get_tuning(wk.PATH_INTRA), "max_ctas": 0, "rate_mbps": r * 1000})
          for r in (50, 150)]),
      "proxy": lambda: bench.run_interference(wk, 0, peaks, configs=[
          (f"push_source_proxy_rate{r}GBs", {**wk.get_tuning(wk.PATH_INTRA), "op": "push_source_proxy",
                                              "max_ctas": 0, "rate_mbps": r * 1000}) for r in (350, 700)] + [
          ("push_source_proxy_uncapped", {**wk.get_tuning(wk.PATH_INTRA), "op": "push_source_proxy",
                                          "max_ctas": 0})]),
      "handoff": lambda: bench.run_handoff(wk, 0),
      "stall_free": lambda: bench.run_stall_free(wk, 0),
      "pressure": lambda: bench.run_pressure(wk, 0),
      "next3": lambda: bench.run_next3(wk, 0, peaks),
      "policy": lambda: bench.run_policy_profile(wk, 0)}[name]
print(json.dumps({name: fn()}))
