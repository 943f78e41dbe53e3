# compute-sanitizer memcheck / racecheck / synccheck on small configs.
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  timeout -s KILL 600 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
     python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/sanitize_smoke_$tool.txt 2>&1
  echo "$tool smoke rc=$? $(tail -1 gpurun_out/sanitize_smoke_$tool.txt)"
done
timeout -s KILL 900 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest -q -x \
  "tests/test_gpu_parity.py::test_migrate_c1_all_kernels" "tests/test_gpu_parity.py::test_run_coalescing_across_warp_windows" \
  "tests/test_gpu_parity.py::test_compact_same_pool" "tests/test_gpu_parity.py::test_swap_round_trip" \
  "tests/test_gpu_heads.py::test_migrate_heads_matches_oracle" > gpurun_out/sanitize_memcheck_tests.txt 2>&1
echo "memcheck tests rc=$? $(tail -2 gpurun_out/sanitize_memcheck_tests.txt | head -1)"
timeout -s KILL 900 compute-sanitizer --tool racecheck --print-limit 20 python -m pytest -q -x \
  "tests/test_gpu_parity.py::test_migrate_c1_all_kernels" "tests/test_gpu_parity.py::test_run_coalescing_across_warp_windows" \
  > gpurun_out/sanitize_racecheck_tests.txt 2>&1
echo "racecheck tests rc=$? $(tail -2 gpurun_out/sanitize_racecheck_tests.txt | head -1)"
# the staged copy-engine swap path (events, side stream, staging buffers)
timeout -s KILL 900 compute-sanitizer --tool memcheck --print-limit 20 python -m pytest -q -x \
  "tests/test_gpu_staged.py" > gpurun_out/sanitize_memcheck_staged.txt 2>&1
echo "memcheck staged rc=$? $(tail -2 gpurun_out/sanitize_memcheck_staged.txt | head -1)"
timeout -s KILL 900 compute-sanitizer --tool racecheck --print-limit 20 python -m pytest -q -x \
  "tests/test_gpu_staged.py::test_staged_round_trip_c1" "tests/test_gpu_staged.py::test_staged_block_chunks_within_a_layer" \
  > gpurun_out/sanitize_racecheck_staged.txt 2>&1
echo "racecheck staged rc=$? $(tail -2 gpurun_out/sanitize_racecheck_staged.txt | head -1)"
