mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
python scripts/plan_info.py 2>&1 | tail -12
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "wide or c5 or random or radix or overlap" > gpurun_out/t_ww.log 2>&1
echo "tests_rc=$?"; tail -3 gpurun_out/t_ww.log
for c in C5a C5b; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --config $c > gpurun_out/b_$c.log 2>&1
  tail -1 gpurun_out/b_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c', 'ms %.3f'%d['ms_per_step'], 'val %.3e'%d['value'], 'scan %.0f GB/s frac %.3f share %.2f grid %s/%s'%(r['achieved'], r['frac'], r['share_of_step'], r['scan_grid'], r['window_grid']))"
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c5a.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --config C5a --tuples-log2 26 > /dev/null 2>&1
python scripts/ncu_summary.py launches gpurun_out/launches_c5a.csv | head -12
