# compute-sanitizer racecheck / synccheck / memcheck on small -m gpu cases:
# shared-memory races, barrier misuse, out-of-bounds accesses.  Logs: gpurun_out/sanitizer/
mkdir -p gpurun_out/sanitizer
export PATH=/usr/local/cuda/bin:$PATH
T="tests/test_gpu_parity.py::test_golden_count tests/test_gpu_parity.py::test_golden_groupby_having_istream tests/test_gpu_parity.py::test_golden_time tests/test_gpu_parity.py::test_random_streams[0] tests/test_gpu_join.py::test_join_windows[sliding_ragged] tests/test_gpu_parity.py::test_bucket_mode[count_only] tests/test_gpu_parity.py::test_win_wide[minmax_having] tests/test_gpu_parity.py::test_time_gap_wider_than_ring[jump1e5_small_ring]"
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
    python -m pytest -m gpu -q -x -p no:cacheprovider $T > gpurun_out/sanitizer/$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitizer/summary.txt
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|passed|failed" gpurun_out/sanitizer/$tool.log | tail -3 >> gpurun_out/sanitizer/summary.txt
done
