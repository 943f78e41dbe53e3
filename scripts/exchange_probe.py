"""Development probe (round 2): full-duplex host swap (swap-out of the C4 victims to one host
pool while another host pool swaps in) on the default SM path, by the swap-out grid size
(bytes of stores in flight into host memory), next to the staged copy-engine path."""
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench  # noqa: E402
import paper_conf_isca_fenghzly025_b200 as wk  # noqa: E402
from windgen import SHAPES  # noqa: E402

sh = SHAPES["C4"]
dev = torch.device("cuda", 0)
nv = 2600  # ~12.7 GiB of C4 blocks (5 MiB each)
dpool = bench.make_pool(wk, sh, nv + 8, 0, 3004, 1)
other = bench.make_pool(wk, sh, nv + 8, 0, 3004, 2)
host = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nv, loc="host")
host2 = wk.Pool(sh.n_layers, sh.n_kv_heads, sh.head_dim, sh.block_size, sh.elem_bytes, nv, loc="host")
vt = torch.as_tensor(np.random.default_rng(1).permutation(nv + 8)[:nv].astype(np.int32), device=dev)
ht = torch.arange(nv, dtype=torch.int32, device=dev)
ht_h = torch.arange(nv, dtype=torch.int32).pin_memory()
s1, s2 = torch.cuda.Stream(dev), torch.cuda.Stream(dev)
vb = bench.payload_bytes(nv, sh.n_layers, sh.chunk_bytes)
saved = wk.get_tuning(wk.PATH_HOST)
out = {}
for name, kern, out_ctas, in_ctas, tab in (("sm_default", wk.KERNEL_AUTO, 0, 0, ht),
                                           ("sm_out4", wk.KERNEL_AUTO, 4, 8, ht),
                                           ("sm_out8", wk.KERNEL_AUTO, 8, 8, ht),
                                           ("sm_out16_in16", wk.KERNEL_AUTO, 16, 16, ht),
                                           ("staged", wk.KERNEL_STAGED, 0, 0, ht_h)):
    def exchange():
        s1.wait_stream(s2)
        wk.migrate_ex(dpool, vt, host2, tab, None if kern == wk.KERNEL_STAGED and False else
                      (wk.tuning(kernel=kern, max_ctas=out_ctas) if kern != wk.KERNEL_AUTO or out_ctas
                       else None), stream=s1)
        wk.migrate_ex(host, tab, other, ht, (wk.tuning(kernel=kern, max_ctas=in_ctas)
                                            if kern != wk.KERNEL_AUTO or in_ctas else None), stream=s2)
        s2.wait_stream(s1)
    try:
        ms = bench.time_device(exchange, 2, 1, s2) / 2
        out[name] = {"aggregate_gbs": round(2 * vb / ms / 1e6, 1), "ms": round(ms, 1)}
    except wk.WindKVError as e:
        out[name] = {"error": str(e)}
    print(name, out[name], flush=True)
wk.set_tuning(wk.PATH_HOST, **saved)
print(json.dumps(out))
