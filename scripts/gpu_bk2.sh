export PATH=/usr/local/cuda/bin:$PATH
run() { tag=$1; G=$2; tm=$3; shift 3
  env "$@" timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e --config C3 --groups $G --task-mb $tm 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$tag G=$G', 'ms %.3f'%d['ms_per_step'], 'scan %.0f'%r['achieved'], r['window_grid'])" || echo "$tag G=$G failed"; }
for G in 1024 4096 16384 65536; do
  tm=1024; [ $G = 16384 ] && tm=512; [ $G = 65536 ] && tm=256
  run base $G $tm X=1
  run sb8k_t256_c2 $G $tm SABER_BK_SB=8192 SABER_BK_THREADS=256 SABER_BK_CTAS=2
  run sb8k_t512_c1 $G $tm SABER_BK_SB=8192
  run sb4k_t256_c3 $G $tm SABER_BK_SB=4096 SABER_BK_THREADS=256 SABER_BK_CTAS=3
done
