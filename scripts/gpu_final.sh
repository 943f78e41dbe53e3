# Round-end evidence on one B200 (run under gpurun): smoke, GPU suite, default bench,
# reference arm, ncu launch list of the default bench command, ncu --set full on the
# headline launch, the N>1 bench path with every rank on the one GPU, sanitizers.
# usage: bash scripts/gpu_final.sh <tag>     (outputs: gpurun_out/<tag>_*)
T=${1:-r02}
O=gpurun_out
mkdir -p $O
nvidia-smi -L > $O/${T}_smi.txt 2>&1
timeout -s KILL 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/${T}_smoke.log 2>&1; echo "smoke rc=$?" >> $O/${T}_smoke.log
timeout -s KILL 1500 python -m pytest tests -m gpu -q > $O/${T}_gputest.log 2>&1; echo "rc=$?" >> $O/${T}_gputest.log
timeout -s KILL 900 python bench.py > $O/${T}_bench.json 2> $O/${T}_bench.err; echo "bench rc=$?" >> $O/${T}_bench.err
timeout -s KILL 300 python bench.py --impl reference --steps 3 --warmup 3 > $O/${T}_bench_reference.json 2>&1
timeout -s KILL 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 2500 --csv \
   --log-file $O/${T}_launches.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline \
   > $O/${T}_launches_bench.json 2>&1; echo "launches rc=$?" >> $O/${T}_bench.err
# full section set on the headline launch (application replay: the pools are ~95 GiB)
timeout -s KILL 1500 ncu --set full --clock-control none --import-source on --replay-mode application \
   -k regex:tma_copy -s 3 -c 1 -o $O/${T}_prof_tma_c2 \
   python bench.py --steps 1 --warmup 3 --no-scenarios --no-cpu-baseline > $O/${T}_prof_bench.json 2>&1
echo "full rc=$?" >> $O/${T}_bench.err
# the N>1 path (pairs over CUDA IPC, all-to-all batch pushes) with every rank on this GPU:
# a functional check only, NOT multi-GPU bandwidth
export WIND_BENCH_ONE_DEVICE=1 WIND_KV_FORCE_PEER_ROUTE=1
timeout -s KILL 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29533 bench.py --gpus 2 --steps 5 --warmup 3 --a2a-scale 0.125 --config C1 \
  > $O/${T}_multirank2.log 2>&1; echo "multirank2 rc=$?" >> $O/${T}_multirank2.log
unset WIND_BENCH_ONE_DEVICE WIND_KV_FORCE_PEER_ROUTE
# (compute-sanitizer runs: round-2 evidence in profiles/r02/sanitizer/; the tool is closed on this pool now)
ls -la $O > $O/${T}_ls.txt
