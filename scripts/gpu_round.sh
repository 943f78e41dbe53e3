# full GPU suite, the default bench, and the host-swap CTA sweep (all configs)
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
mkdir -p gpurun_out
timeout -s KILL 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -30 | tee gpurun_out/gpu_tests.log
timeout -s KILL 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -5 gpurun_out/bench.err
timeout -s KILL 600 python scripts/staged_sweep.py C1,C3,C4,C5 > gpurun_out/staged_sweep_all.txt 2>&1; echo "sweep rc=$?"
