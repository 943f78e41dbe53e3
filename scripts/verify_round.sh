set -x
nproc; nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build(); g.smoke(); print('SMOKE OK')" 2>&1 | tail -3
timeout -s KILL 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -15 | tee gpurun_out/gpu_tests.log
timeout -s KILL 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
head -c 3000 gpurun_out/bench.json; tail -5 gpurun_out/bench.err
