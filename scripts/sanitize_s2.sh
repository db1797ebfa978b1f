# compute-sanitizer on the round-2 session-2 kernels (k_pane_cnt CTA table / owned panes /
# bitmaps, k_wb_rows, k_win_block_reg incl. key slices, k_bkt_rows, k_join_emit_i32, the
# time-window CTA table): small -m gpu cases.  Logs: gpurun_out/sanitizer_s2/
mkdir -p gpurun_out/sanitizer_s2
export PATH=/usr/local/cuda/bin:$PATH
T="tests/test_gpu_parity.py::test_win_block_reg[c64_k16] tests/test_gpu_parity.py::test_win_block_reg[c256_k32] tests/test_gpu_parity.py::test_win_block_reg[time_c64_k32] tests/test_gpu_parity.py::test_golden_count tests/test_gpu_join.py::test_join_windows[sliding_ragged]"
for tool in memcheck racecheck synccheck; do
  timeout 2400 compute-sanitizer --tool $tool --target-processes all --print-limit 20 \
    python -m pytest -m gpu -q -x -p no:cacheprovider $T > gpurun_out/sanitizer_s2/$tool.log 2>&1
  echo "$tool rc=$?" >> gpurun_out/sanitizer_s2/summary.txt
  grep -E "ERROR SUMMARY|RACECHECK SUMMARY|passed|failed" gpurun_out/sanitizer_s2/$tool.log | tail -3 >> gpurun_out/sanitizer_s2/summary.txt
done
