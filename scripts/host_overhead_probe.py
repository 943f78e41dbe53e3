"""Development probe (round 2): host-side cost of enqueueing an op (no blocking on the
hot path) — wall time per wind_kv_migrate call from Python (ctypes marshalling + argument
checks + launch) and per raw C-ABI call (ctypes, pre-marshalled arguments), for 400 ops
queued behind a sleeping kernel so the GPU never drains the queue mid-measurement."""
import ctypes as ct
import json
import os
import sys
import time

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402

dev = torch.device("cuda", 0)
src = wk.Pool(40, 40, 128, 16, 2, 64)
dst = wk.Pool(40, 40, 128, 16, 2, 64)
ts = torch.arange(4, dtype=torch.int32, device=dev)
td = torch.arange(8, 12, dtype=torch.int32, device=dev)
s = torch.cuda.Stream(dev)
out = {}
for name in ("python_binding", "raw_c_abi"):
    for _ in range(2):
        torch.cuda.synchronize()
        with torch.cuda.stream(s):
            torch.cuda._sleep(50_000_000)
        L = wk.lib()
        args = (src.handle, ts.data_ptr(), dst.handle, td.data_ptr(), 4, 0, 40, s.cuda_stream)
        t0 = time.perf_counter()
        if name == "python_binding":
            for _ in range(400):
                wk.migrate(src, ts, dst, td, stream=s)
        else:
            f = L.wind_kv_migrate
            for _ in range(400):
                f(*args)
        t1 = time.perf_counter()
        torch.cuda.synchronize()
    out[f"{name}_us_per_call"] = round((t1 - t0) / 400 * 1e6, 2)
print(json.dumps(out))
