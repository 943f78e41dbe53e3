"""Development helper: the C1 intra-device migrate (144 MiB, L2 flushed before each op) and a
1-block op (fixed cost) under several launch tunings."""
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
case = migration_case(sys.argv[1] if len(sys.argv) > 1 else "C1")
sh = case.shape
a = bench.make_pool(wk, sh, case.nb_src, 0, case.content_seed, case.src_tag)
b = bench.make_pool(wk, sh, case.nb_dst, 0, case.content_seed, case.dst_tag)
sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
flush = torch.ones(2 * (126 << 20) // 4, dtype=torch.int32, device=dev)
s = torch.cuda.Stream(dev)
pb = bench.payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)


def timed(fn, reps=30):
    for _ in range(3):
        fn()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(reps)]
    torch.cuda.synchronize()
    with torch.cuda.stream(s):
        for e0, e1 in ev:
            flush.sum(dtype=torch.int64)
            e0.record(s)
            fn()
            e1.record(s)
    torch.cuda.synchronize()
    return float(np.median([e0.elapsed_time(e1) for e0, e1 in ev]))


T = wk.KERNEL_TMA
out = {}
if "--graph" in sys.argv:
    for n_ in (case.n, 1):
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            wk.migrate(a, sbt[:n_], b, dbt[:n_], stream=s)
        torch.cuda.synchronize()
        ms = timed(g.replay)
        pbn = bench.payload_bytes(n_, sh.n_layers, sh.chunk_bytes)
        # back to back, no flush: 20 replays between two events
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            ev0.record(s)
            for _ in range(20):
                g.replay()
            ev1.record(s)
        torch.cuda.synchronize()
        out[f"graph_n{n_}"] = {"gbs": round(pbn / ms / 1e6, 1), "us_flushed": round(ms * 1e3, 2),
                               "us_back_to_back": round(ev0.elapsed_time(ev1) / 20 * 1e3, 2)}
        print(f"graph_n{n_}", out[f"graph_n{n_}"], flush=True)
for name, t in [("default", None),
                ("u24k_s8", wk.tuning(kernel=T, stage_bytes=24576, stages=8, store_lag=4)),
                ("u48k_s4_lag1", wk.tuning(kernel=T, stage_bytes=49152, stages=4, store_lag=1)),
                ("u48k_s4_lag3", wk.tuning(kernel=T, stage_bytes=49152, stages=4, store_lag=3)),
                ("u96k_s2", None),
                ("u16k_s12_lag6", wk.tuning(kernel=T, stage_bytes=16384, stages=12, store_lag=6)),
                ("u48k_s4_2cta", wk.tuning(kernel=T, stage_bytes=49152, stages=4, store_lag=2, ctas_per_sm=2)),
                ("u24k_s4_2cta", wk.tuning(kernel=T, stage_bytes=24576, stages=4, store_lag=2, ctas_per_sm=2)),
                ("simt_4cta_32k", wk.tuning(kernel=wk.KERNEL_SIMT, stage_bytes=32768, stages=4, ctas_per_sm=4)),
                ("simt_4cta_8k", wk.tuning(kernel=wk.KERNEL_SIMT, stage_bytes=8192, stages=4, ctas_per_sm=4))]:
    if name == "u96k_s2":
        continue
    ms = timed(lambda: wk.migrate_ex(a, sbt, b, dbt, t, stream=s))
    ms1 = timed(lambda: wk.migrate_ex(a, sbt[:1], b, dbt[:1], t, stream=s))
    out[name] = {"gbs": round(pb / ms / 1e6, 1), "ms": round(ms, 4), "one_block_us": round(ms1 * 1e3, 2)}
    print(name, out[name], flush=True)
print(json.dumps(out))
