"""Probe: does a migration on stream A delay a tiny kernel on stream B?  (copy-engine
paced / unpaced, TMA rate-limited).  Development tool."""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
import windgen.cuda as wg  # noqa: E402
from windgen import SHAPES  # noqa: E402

dev = torch.device("cuda", 0)
sh = SHAPES["C2"]
nb = 400
src = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
dst = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, 16, 2, nb)
wg.fill(src.base, src.nbytes, 0, 1, 1)
perm = np.random.default_rng(0).permutation(nb)[:128].astype(np.int32)
hs = torch.as_tensor(perm).pin_memory()
ds = torch.as_tensor(perm, device=dev)
a, b = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
x = torch.zeros(1024, device=dev)
with torch.cuda.stream(b):
    x.add_(1)  # warm: load the tiny kernel's module before any migration runs
torch.cuda.synchronize()
res = {}
for name, tun, tab in [("ce_paced_200", wk.tuning(kernel=3, rate_mbps=200_000), hs.data_ptr()),
                       ("ce_unpaced", wk.tuning(kernel=3), hs.data_ptr()),
                       ("tma_rate_200", wk.tuning(rate_mbps=200_000), ds.data_ptr()),
                       ("none", None, None)]:
    torch.cuda.synchronize()
    if tun is not None:
        for _ in range(3):
            wk.migrate_ex(src, tab, dst, tab, tun, n=128, stream=a)
    ev = torch.cuda.Event()
    ev.record(a)
    lat = []
    for _ in range(20):
        t0 = time.perf_counter()
        with torch.cuda.stream(b):
            x.add_(1)
        b.synchronize()
        lat.append((time.perf_counter() - t0) * 1e3)
    busy = not ev.query()
    torch.cuda.synchronize()
    res[name] = {"tiny_kernel_ms_median": round(float(np.median(lat)), 3),
                 "tiny_kernel_ms_max": round(max(lat), 3), "migration_still_running": busy}
print(json.dumps(res), os.environ.get("CUDA_DEVICE_MAX_CONNECTIONS"))
