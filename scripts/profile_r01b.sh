# Refreshed ncu evidence after the GPU-scope publication change (run under gpurun; one GPU).
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
mkdir -p gpurun_out
timeout -s KILL 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 2500 --csv \
   --log-file gpurun_out/launches_bench_v2.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline \
   > gpurun_out/launches_bench_v2.json 2>&1
echo "launches rc=$?"
timeout -s KILL 1500 ncu --set full --clock-control none --import-source on --replay-mode application \
   -k regex:tma_copy -s 3 -c 1 -o gpurun_out/prof_tma_c2_v2 \
   python bench.py --steps 1 --warmup 3 --no-scenarios --no-cpu-baseline > gpurun_out/prof_c2_v2.log 2>&1
echo "full c2 rc=$?"
timeout -s KILL 900 ncu --set full --clock-control none --import-source on \
   -k regex:tma_copy -s 3 -c 1 -o gpurun_out/prof_compact_v2 python scripts/overhead_probe.py \
   > gpurun_out/prof_compact_v2.log 2>&1
echo "full compact rc=$?"
bash scripts/sanitize.sh
