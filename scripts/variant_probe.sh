# Runs scripts/overhead_probe.py against each library variant scratch_v*/ (development).
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
LIB=paper_conf_isca_fenghzly025_b200/libwind_kv.so
cp $LIB /tmp/cur.so
for d in scratch_v*; do
  cp $d/libwind_kv.so $LIB
  echo "== $d"
  timeout -s KILL 300 python scripts/overhead_probe.py 2>&1 | grep -v "size\"" | grep -E "compact|one_block|sequential\"|shuffled_both"
done
cp /tmp/cur.so $LIB
