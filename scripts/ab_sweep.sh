# A/B of the copy kernels: the working tree's library vs a saved one (scratch_old/).
# usage (under gpurun): bash scripts/ab_sweep.sh <modes...>
set -u
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
mkdir -p gpurun_out
LIB=paper_conf_isca_fenghzly025_b200/libwind_kv.so
cp $LIB /tmp/new.so
for tag in new old new2; do
  if [ $tag = old ]; then cp scratch_old/libwind_kv.so $LIB; else cp /tmp/new.so $LIB; fi
  for m in "$@"; do
    timeout -s KILL 600 python scripts/sweep.py $m > gpurun_out/sw_${tag}_$m.txt 2>&1
  done
done
cp /tmp/new.so $LIB
