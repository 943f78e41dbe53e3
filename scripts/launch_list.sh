# ncu launch list of the default bench command (first 2500 launches: the headline step and
# the first scenarios; later launches run unprofiled).  usage: bash scripts/launch_list.sh <tag>
TAG=${1:-r01}
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
mkdir -p gpurun_out
timeout -s KILL 1500 ncu --metrics gpu__time_duration.sum --clock-control none -c 2500 --csv \
   --log-file gpurun_out/launches_$TAG.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline \
   > gpurun_out/launches_bench_$TAG.json 2>&1
echo "launches rc=$?"
