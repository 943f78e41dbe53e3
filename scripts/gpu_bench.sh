python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout -s KILL 900 python -m pytest tests/test_gpu_victim.py tests/test_gpu_parity.py -q -x 2>&1 | tail -5
timeout -s KILL 900 python bench.py "$@" > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json; tail -5 gpurun_out/bench.err
