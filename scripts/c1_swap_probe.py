import json, os, sys
sys.path.insert(0, os.getcwd())
import torch, bench
import paper_conf_isca_fenghzly025_b200 as wk
from windgen import migration_case
dev = torch.device("cuda", 0)
case = migration_case("C1"); sh1 = case.shape
dpool = bench.make_pool(wk, sh1, case.nb_src, 0, case.content_seed, case.src_tag)
dpool2 = bench.make_pool(wk, sh1, case.nb_dst, 0, case.content_seed, case.dst_tag)
hpool = wk.Pool(sh1.n_layers, sh1.n_kv_heads, sh1.head_dim, sh1.block_size, sh1.elem_bytes, case.n, loc="host")
hbt_h = torch.arange(case.n, dtype=torch.int32).pin_memory()
hbt = torch.arange(case.n, dtype=torch.int32, device=dev)
sbt = torch.as_tensor(case.src_bt, device=dev)
pb = bench.payload_bytes(case.n, sh1.n_layers, sh1.chunk_bytes)
s = torch.cuda.Stream(dev)
for rep in range(2):
    for mech, ht in (("sm", hbt), ("staged", hbt_h), ("sm", hbt)):
        for steps in (3, 10):
            ms = bench.time_device(lambda: wk.swap_out(dpool, sbt, hpool, ht, stream=s), steps, 3, s) / steps
            print(rep, mech, steps, round(pb / ms / 1e6, 2), flush=True)
    ms = bench.time_device(lambda: wk.swap_out(dpool, sbt, hpool, hbt, stream=s), 10, 3, s, per_step=(ps := [])) / 10
    print("per-step ms", [round(x, 3) for x in ps])
