mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
for v in base ${VARIANTS}; do
  if [ $v = base ]; then lib=""; else lib=$PWD/build_var/$v.so; fi
  for c in ${CONFIGS:-C3}; do
    SABER_LIB=$lib timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --config $c $EXTRA > gpurun_out/bv_${v}_$c.log 2>&1
    tail -1 gpurun_out/bv_${v}_$c.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$v $c', 'ms %.3f'%d['ms_per_step'], 'val %.3e'%d['value'], 'scan %.0f GB/s frac %.3f share %.2f grid %s/%s'%(r['achieved'], r['frac'], r['share_of_step'], r['scan_grid'], r['window_grid']))" || tail -3 gpurun_out/bv_${v}_$c.log
  done
done
