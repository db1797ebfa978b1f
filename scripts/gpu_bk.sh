export PATH=/usr/local/cuda/bin:$PATH
for G in 256 512 1024 2048 4096; do
 for nb in 0 1; do
  SABER_NO_BUCKET=$nb timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e --config C3 --groups $G --task-mb 1024 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('G=$G nobucket=$nb', 'ms %.3f'%d['ms_per_step'], 'scan %.0f'%r['achieved'], r['kernel'], r['window_kernels'], r['scan_grid'], r['window_grid'])" || echo "G=$G nb=$nb failed"
 done
done
