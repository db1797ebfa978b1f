# all GPU tests, the default bench line, and a launch list of one config (1 GPU)
mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/t_all.log 2>&1
echo "tests_rc=$?"; tail -3 gpurun_out/t_all.log
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e ${BENCH_ARGS} > gpurun_out/bench_main.log 2>&1
tail -1 gpurun_out/bench_main.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('value',d['value'],'ms',d['ms_per_step'],'frac',d['roofline']['frac'],'scan GB/s',d['roofline']['achieved'],'clk',d['clocks'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_main.csv python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu ${LAUNCH_ARGS} > /dev/null 2>&1
python scripts/ncu_summary.py launches gpurun_out/launches_main.csv > gpurun_out/l.txt; head -9 gpurun_out/l.txt
