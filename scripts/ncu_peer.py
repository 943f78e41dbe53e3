"""ncu target for the NVLink evidence (needs >= 2 GPUs in ONE process, so ncu can replay the
kernel): C2-geometry pools on cuda:0 and cuda:1, a push 0 -> 1 (executes on 0, peer stores
into 1) and a push 1 -> 0, 500 blocks, each launched 4 + 1 times.  (A pull needs the source
pool imported from another process: the bench's N > 1 autotune times it.)
Profile, e.g.:
  ncu --clock-control none --metrics gpu__time_duration.sum,nvltx__bytes_data_user.sum,\
nvlrx__bytes_data_user.sum,dram__bytes_read.sum,dram__bytes_write.sum \
      -k regex:"tma_copy|simt_copy" python scripts/ncu_peer.py [tma|simt]
Without ncu it prints the CUDA-event rate of each direction."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
from windgen import SHAPES  # noqa: E402

if torch.cuda.device_count() < 2:
    raise SystemExit("needs 2 GPUs")
kern = {"tma": wk.KERNEL_TMA, "simt": wk.KERNEL_SIMT}[sys.argv[1] if len(sys.argv) > 1 else "simt"]
sh = SHAPES["C2"]
n, nb = 500, 560
a = bench.make_pool(wk, sh, nb, 0, 1, 1)
b = bench.make_pool(wk, sh, nb, 1, 1, 2)
rng = np.random.default_rng(0)
sbt, dbt = rng.permutation(nb)[:n].astype(np.int32), rng.permutation(nb)[:n].astype(np.int32)
wk.set_tuning(wk.PATH_PEER, kernel=kern, ctas_per_sm=4 if kern == wk.KERNEL_SIMT else 1)
pb = bench.payload_bytes(n, sh.n_layers, sh.chunk_bytes)
for name, src, dst in (("push 0->1", a, b), ("push 1->0", b, a)):
    s = torch.cuda.Stream(device=src.device)
    st = torch.as_tensor(sbt, device=torch.device("cuda", src.device))
    dt = torch.as_tensor(dbt, device=torch.device("cuda", src.device))
    e, p, scope = wk.route(src, dst)
    ms = bench.time_device(lambda: wk.migrate(src, st, dst, dt, stream=s), 4, 1, s) / 4
    print(f"{name}: executes on {e}, path {p}, sys scope {scope}: {pb / ms / 1e6:.1f} GB/s", flush=True)
