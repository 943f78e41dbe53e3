"""Development probe: the default-tuning small ops of bench c1_intra (C1 migrate, C1
compaction, a 1-block op), each timed alone between two CUDA events after an L2 flush, and
20 compactions back to back.  Used to A/B library builds (run from each build's tree).
Usage: python scripts/small_op_ab.py <label>"""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
from windgen import migration_case, live_mask_after_free, request_lengths, blocks_for_tokens  # noqa: E402

dev = torch.device("cuda", 0)
case = migration_case("C1")
sh = case.shape
a = bench.make_pool(wk, sh, case.nb_src, 0, case.content_seed, case.src_tag)
b = bench.make_pool(wk, sh, case.nb_dst, 0, case.content_seed, case.dst_tag)
sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
reqb = blocks_for_tokens(request_lengths("C1"), sh.block_size)
live, _ = live_mask_after_free(case.nb_src, reqb, 0.5, 4001)
csrc, cdst = wk.plan_compact(live)
ts, td = torch.as_tensor(csrc, device=dev), torch.as_tensor(cdst, device=dev)
flush = torch.ones(2 * (126 << 20) // 4, dtype=torch.int32, device=dev)
s = torch.cuda.Stream(dev)


def timed(fn, reps=100):
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
    return float(np.median([e0.elapsed_time(e1) for e0, e1 in ev])) * 1e3


r = {"label": sys.argv[1] if len(sys.argv) > 1 else ""}
r["migrate_us"] = round(timed(lambda: wk.migrate(a, sbt, b, dbt, stream=s)), 2)
r["compact_us"] = round(timed(lambda: wk.migrate(a, ts, a, td, stream=s)), 2)
r["one_block_us"] = round(timed(lambda: wk.migrate(a, sbt[:1], b, dbt[:1], stream=s)), 2)
ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
with torch.cuda.stream(s):
    ev0.record(s)
    for _ in range(50):
        wk.migrate(a, ts, a, td, stream=s)
    ev1.record(s)
torch.cuda.synchronize()
r["compact_b2b_us"] = round(ev0.elapsed_time(ev1) / 50 * 1e3, 2)
print(json.dumps(r), flush=True)
