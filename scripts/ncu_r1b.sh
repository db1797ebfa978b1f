mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_r1b.csv python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu > /dev/null 2>&1
echo rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pane_agg -s 4 -c 1 -o gpurun_out/prof_pane2 python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu > /dev/null 2>&1
echo rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_vh_build|k_win_vh" -s 6 -c 3 -o gpurun_out/prof_win2 python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu > /dev/null 2>&1
echo rc=$?
