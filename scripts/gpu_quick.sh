# quick bench of selected configs: CONFIGS="C5a C5b" bash scripts/gpu_quick.sh
mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
for c in ${CONFIGS:-C3 C5a C5b}; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --config $c $EXTRA > gpurun_out/b_$c.log 2>&1
  tail -1 gpurun_out/b_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c', 'ms %.3f'%d['ms_per_step'], 'val %.3e'%d['value'], 'scan %.0f GB/s frac %.3f share %.2f grid %s/%s'%(r['achieved'], r['frac'], r['share_of_step'], r['scan_grid'], r['window_grid']))" || tail -5 gpurun_out/b_$c.log
done
if [ -n "$LAUNCH" ]; then
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_q.csv python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu --config $LAUNCH --tuples-log2 26 > /dev/null 2>&1
python scripts/ncu_summary.py launches gpurun_out/launches_q.csv | head -12
fi
