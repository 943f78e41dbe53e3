# round-end evidence: smoke, GPU suite, default bench, ncu launch list of the default bench
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('SMOKE OK')" 2>&1 | tail -2
mkdir -p gpurun_out
timeout -s KILL 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -5 | tee gpurun_out/gpu_tests.log
timeout -s KILL 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -3 gpurun_out/bench.err
timeout -s KILL 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_reference.json 2>&1; echo "ref rc=$?"
timeout -s KILL 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 2500 --csv \
   --log-file gpurun_out/launches_final.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline \
   > gpurun_out/launches_bench_final.json 2>&1
echo "launches rc=$?"
# full section set on the headline launch (application replay: the pools are ~95 GiB)
timeout -s KILL 1500 ncu --set full --clock-control none --import-source on --replay-mode application \
   -k regex:tma_copy -s 3 -c 1 -o gpurun_out/prof_tma_c2_final \
   python bench.py --steps 1 --warmup 3 --no-scenarios --no-cpu-baseline > gpurun_out/prof_bench_final.json 2>&1
echo "full rc=$?"
