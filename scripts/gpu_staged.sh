# staged copy-engine swap path: its parity tests, the full GPU suite, the default bench
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
mkdir -p gpurun_out
timeout -s KILL 600 python -m pytest tests/test_gpu_staged.py -q -x 2>&1 | tail -30 | tee gpurun_out/staged_tests.log
timeout -s KILL 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -30 | tee gpurun_out/gpu_tests.log
timeout -s KILL 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -5 gpurun_out/bench.err
