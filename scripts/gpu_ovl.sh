# overlap experiment: GPU tests + default bench with/without overlap and grid variants
mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/t_all.log 2>&1
echo "tests_rc=$?"; tail -3 gpurun_out/t_all.log
b() { tag=$1; shift
  env "$@" timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e ${BENCH_ARGS} > gpurun_out/b_$tag.log 2>&1
  tail -1 gpurun_out/b_$tag.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$tag', 'ms %.3f'%d['ms_per_step'], 'val %.3e'%d['value'], 'scan %.0f GB/s frac %.3f share %.2f'%(r['achieved'], r['frac'], r['share_of_step']), d['clocks']['sm_mhz'], d['clocks']['reasons'])" 2>&1 | tail -1
}
b noovl SABER_NO_OVERLAP=1
b ovl_s3w1 SABER_OVL_SCAN_BPS=3 SABER_OVL_WIN_BPS=1
b ovl_s4w1 SABER_OVL_SCAN_BPS=4 SABER_OVL_WIN_BPS=1
b ovl_s2w1 SABER_OVL_SCAN_BPS=2 SABER_OVL_WIN_BPS=1
b ovl_s3w2 SABER_OVL_SCAN_BPS=3 SABER_OVL_WIN_BPS=2
for c in C4 C5a C5b SG1 C1; do
  BENCH_ARGS="--config $c" b ${c}_noovl SABER_NO_OVERLAP=1
  BENCH_ARGS="--config $c" b ${c}_ovl X=1
done
