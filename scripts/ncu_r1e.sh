mkdir -p gpurun_out/r1e
export PATH=/usr/local/cuda/bin:$PATH
for kb in 48 24; do
for c in C5a C5b; do
  SABER_SHARED_KB=$kb timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --config $c > gpurun_out/r1e/b_${c}_$kb.log 2>&1
  tail -1 gpurun_out/r1e/b_${c}_$kb.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('$c $kb', 'ms %.3f'%d['ms_per_step'], 'val %.3e'%d['value'], 'scan %.0f GB/s frac %.3f share %.2f grid %s/%s'%(r['achieved'], r['frac'], r['share_of_step'], r['scan_grid'], r['window_grid']))"
done; done
full() { tag=$1; kre=$2; skip=$3; shift 3
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$kre -s $skip -c 1 -o gpurun_out/r1e/prof_$tag \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > /dev/null 2>&1
  python scripts/ncu_summary.py report gpurun_out/r1e/prof_$tag.ncu-rep --json gpurun_out/r1e/ncu_full_$tag.json > gpurun_out/r1e/sum_$tag.txt 2>&1; echo "$tag done"; }
full k_win_wide_C5a k_win_wide 4 --config C5a --tuples-log2 26
full k_vh_build_tile_C5a k_vh_build_tile 4 --config C5a --tuples-log2 26
