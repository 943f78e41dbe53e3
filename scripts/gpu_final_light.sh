# round-end check without the ncu passes: smoke, GPU suite, default bench, reference arm
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
mkdir -p gpurun_out
timeout -s KILL 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 | tee gpurun_out/gpu_tests.log
timeout -s KILL 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -2 gpurun_out/bench.err
timeout -s KILL 300 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_reference.json 2>&1; echo "ref rc=$?"
