mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
for tm in 512 1024 2048 4096 8192; do
  timeout 300 python bench.py --steps 8 --warmup 3 --no-cpu --no-e2e --config C3 --task-mb $tm > gpurun_out/b_t$tm.log 2>&1
  tail -1 gpurun_out/b_t$tm.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$tm', 'ms %.3f'%d['ms_per_step'], 'val %.3e'%d['value'], 'scan %.0f GB/s frac %.3f share %.2f grid %s/%s'%(r['achieved'], r['frac'], r['share_of_step'], r['scan_grid'], r['window_grid']))" || tail -3 gpurun_out/b_t$tm.log
done
for tm in 1024 4096; do
  SABER_OVERLAP=1 timeout 300 python bench.py --steps 8 --warmup 3 --no-cpu --no-e2e --config C3 --task-mb $tm > gpurun_out/b_o$tm.log 2>&1
  tail -1 gpurun_out/b_o$tm.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('ovl $tm', 'ms %.3f'%d['ms_per_step'], 'val %.3e'%d['value'], 'scan %.0f GB/s frac %.3f share %.2f grid %s/%s'%(r['achieved'], r['frac'], r['share_of_step'], r['scan_grid'], r['window_grid']))" || tail -3 gpurun_out/b_o$tm.log
done
