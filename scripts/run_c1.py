"""Development helper: bench.py's C1 intra-device scenario alone (single-op and
stream-of-cold-ops numbers), printed as one JSON line."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402

peaks = bench.load_peaks() if hasattr(bench, "load_peaks") else {"hbm_gbs": 6553.3}
print(json.dumps(bench.run_c1_intra(wk, 0, peaks)))
