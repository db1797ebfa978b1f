mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
python scripts/plan_info.py 2>&1 | tail -12
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/t_all.log 2>&1
echo "tests_rc=$?"; tail -3 gpurun_out/t_all.log
for c in C5a C5b SG1 C4; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --config $c > gpurun_out/b_$c.log 2>&1
  tail -1 gpurun_out/b_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c', 'ms %.3f'%d['ms_per_step'], 'val %.3e'%d['value'], 'scan %.0f GB/s frac %.3f share %.2f grid %s/%s'%(r['achieved'], r['frac'], r['share_of_step'], r['scan_grid'], r['window_grid']))"
done
