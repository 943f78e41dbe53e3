"""Development helper: staged swap rate vs the CTA count of the hidden gather / scatter
chunks, C1 and C3 geometries, standalone (no co-running work)."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
from windgen import migration_case  # noqa: E402

dev = torch.device("cuda", 0)
CFGS = sys.argv[1].split(",") if len(sys.argv) > 1 else ["C1", "C3", "C5"]
out = {}
for cfg, nsw in [(c, n) for c, n in (("C1", None), ("C3", 64), ("C4", 400), ("C5", 4096)) if c in CFGS]:
    case = migration_case(cfg)
    sh = case.shape
    n = int(os.environ.get("STAGED_N", 0)) or nsw or case.n
    n = min(n, case.n)
    src = bench.make_pool(wk, sh, case.nb_src, 0, case.content_seed, case.src_tag)
    host = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, n, loc="host")
    sbt = torch.as_tensor(case.src_bt[:n], device=dev)
    hh = torch.arange(n, dtype=torch.int32).pin_memory()
    hd = torch.arange(n, dtype=torch.int32, device=dev)
    pb = bench.payload_bytes(n, sh.n_layers, sh.chunk_bytes)
    s = torch.cuda.Stream(dev)
    saved = wk.get_tuning(wk.PATH_HOST)
    r = {}
    for name, ht, c in [("staged_auto", hh, dict(kernel=4, max_ctas=0)), ("sm_auto", hd, dict(kernel=1, max_ctas=0)),
                        ("staged_h1", hh, dict(kernel=4, max_ctas=1)), ("staged_h2", hh, dict(kernel=4, max_ctas=2)),
                        ("staged_h4", hh, dict(kernel=4, max_ctas=4)), ("staged_h8", hh, dict(kernel=4, max_ctas=8)),
                        ("staged_h32", hh, dict(kernel=4, max_ctas=32)), ("staged_h148", hh, dict(kernel=4, max_ctas=148)),
                        ("sm_tma1", hd, dict(kernel=1, max_ctas=1)), ("sm_tma2", hd, dict(kernel=1, max_ctas=2)),
                        ("sm_tma3", hd, dict(kernel=1, max_ctas=3)), ("sm_simt2", hd, dict(kernel=2, max_ctas=2)),
                        ("sm_tma4", hd, dict(kernel=1, max_ctas=4)), ("sm_tma8", hd, dict(kernel=1, max_ctas=8))]:
        wk.set_tuning(wk.PATH_HOST, **{**saved, **c})
        to = bench.time_device(lambda: wk.swap_out(src, sbt, host, ht, stream=s), 3, 3, s) / 3
        ti = bench.time_device(lambda: wk.swap_in(host, ht, src, sbt, stream=s), 3, 3, s) / 3
        r[name] = (round(pb / to / 1e6, 2), round(pb / ti / 1e6, 2))
    wk.set_tuning(wk.PATH_HOST, **saved)
    out[cfg] = {"blocks": n, "payload_mib": round(pb / 2**20, 1), "out_in_gbs": r}
    print(cfg, json.dumps(out[cfg]), flush=True)
    host.destroy()
    del src
    torch.cuda.empty_cache()
print(json.dumps(out))
