set -x
mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1.csv python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu > gpurun_out/ncu_launch_bench.log 2>&1
echo rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pane_agg -s 4 -c 1 -o gpurun_out/prof_pane python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu > gpurun_out/ncu_full_pane.log 2>&1
echo rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_win_dense -s 8 -c 2 -o gpurun_out/prof_win python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu > gpurun_out/ncu_full_win.log 2>&1
echo rc=$?
ls -la gpurun_out
