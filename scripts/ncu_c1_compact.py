"""ncu target: the C1 compaction op (67 moves, 39.5 MB) and a 1-block C1 migrate, each
after an L2 flush, a few times (profile with -k regex:tma_copy -s <skip> -c 1)."""
import os
import sys

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
reqb = blocks_for_tokens(request_lengths("C1"), sh.block_size)
live, _ = live_mask_after_free(case.nb_src, reqb, 0.5, 4001)
csrc, cdst = wk.plan_compact(live)
ts, td = torch.as_tensor(csrc, device=dev), torch.as_tensor(cdst, device=dev)
sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
flush = torch.ones(2 * (126 << 20) // 4, dtype=torch.int32, device=dev)
which = sys.argv[1] if len(sys.argv) > 1 else "compact"
for _ in range(4):
    flush.sum(dtype=torch.int64)
    if which == "compact":
        wk.compact(a, ts, td)
    else:
        wk.migrate(a, sbt[:1], b, dbt[:1])
torch.cuda.synchronize()
print("done", which)
