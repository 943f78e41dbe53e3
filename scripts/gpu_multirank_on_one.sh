# Exercise the N>1 bench path (pairs over CUDA IPC, all-to-all batch pushes into imported
# pools) with every rank on the one GPU of a gpurun box.  Test hook only: numbers printed
# here are NOT multi-GPU bandwidth (all ranks share one HBM).
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
export WIND_BENCH_ONE_DEVICE=1
timeout -s KILL 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --a2a-scale 0.125 --config C1 2>&1 | tail -5
timeout -s KILL 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 3 --master-addr 127.0.0.1 \
  --master-port 29534 bench.py --gpus 3 --steps 5 --warmup 3 --a2a-scale 0.125 --config C1 2>&1 | tail -5
timeout -s KILL 300 python bench.py --impl reference --steps 3 --warmup 3 2>&1 | tail -2
