python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
mkdir -p gpurun_out
timeout -s KILL 900 ncu --set full --clock-control none --import-source on -k regex:"simt_copy|decode_split" \
  -s 1 -c 2 -o gpurun_out/prof_secondary python scripts/ncu_targets.py > gpurun_out/prof_secondary.log 2>&1
echo "rc=$?"; tail -3 gpurun_out/prof_secondary.log
