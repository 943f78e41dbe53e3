# ncu evidence for the bench's dominant kernel (run under gpurun; one GPU).
# usage: bash scripts/profile.sh <tag>
TAG=${1:-r01}
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
mkdir -p gpurun_out
# 1) launch list of the bench command (cold-cache, serialised: compare shares)
timeout -s KILL 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline \
   > gpurun_out/launches_bench_$TAG.json 2>&1
echo "launches rc=$?"
# 2) full section set on one tma_copy_kernel launch of the C2 step (application replay:
#    the 95 GiB of pools are too large to save/restore per kernel replay)
timeout -s KILL 1500 ncu --set full --clock-control none --import-source on --replay-mode application \
   -k regex:tma_copy -s 3 -c 1 -o gpurun_out/prof_tma_c2_$TAG \
   python bench.py --steps 1 --warmup 3 --no-scenarios --no-cpu-baseline > gpurun_out/prof_bench_$TAG.json 2>&1
echo "full rc=$?"
ls -la gpurun_out
