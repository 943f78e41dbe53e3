python -c "import __graft_entry__ as g; g.build()" >/dev/null 2>&1
timeout -s KILL 1200 python -m pytest tests -m gpu -q -x 2>&1 | tail -2
for P in 1 0 1 0; do
  echo "PDL=$P"
  WIND_KV_PDL=$P timeout -s KILL 300 python - <<'PY'
import os, sys, json
sys.path.insert(0, os.getcwd())
import torch, bench
import paper_conf_isca_fenghzly025_b200 as wk
from windgen import migration_case
dev = torch.device("cuda", 0)
case = migration_case("C2"); sh = case.shape
src = bench.make_pool(wk, sh, case.nb_src, 0, case.content_seed, case.src_tag)
dst = bench.make_pool(wk, sh, case.nb_dst, 0, case.content_seed, case.dst_tag)
sbt, dbt = torch.as_tensor(case.src_bt, device=dev), torch.as_tensor(case.dst_bt, device=dev)
s = torch.cuda.Stream(dev)
pb = bench.payload_bytes(case.n, sh.n_layers, sh.chunk_bytes)
def streamed():
    for l in range(sh.n_layers):
        wk.migrate(src, sbt, dst, dbt, layer_lo=l, layer_hi=l + 1, stream=s)
ms = bench.time_device(streamed, 10, 3, s) / 10
one = bench.time_device(lambda: wk.migrate(src, sbt[:1], dst, dbt[:1], stream=s), 200, 10, s) / 200
print(json.dumps({"streamed_gbs": round(pb / ms / 1e6, 1), "streamed_ms": round(ms, 3), "one_block_back_to_back_us": round(one * 1e3, 2)}))
PY
done
