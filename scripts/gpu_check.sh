set -x
nvidia-smi --query-gpu=name,memory.total,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -5
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -20
timeout -s KILL 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -40
timeout -s KILL 600 python bench.py --steps 20 --warmup 3 > gpurun_out/bench1.json 2> gpurun_out/bench1.err; echo bench rc=$?
tail -c 3000 gpurun_out/bench1.json; tail -20 gpurun_out/bench1.err
