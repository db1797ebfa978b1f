mkdir -p gpurun_out/r1d
export PATH=/usr/local/cuda/bin:$PATH
full() { tag=$1; kre=$2; skip=$3; shift 3
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$kre -s $skip -c 1 -o gpurun_out/r1d/prof_$tag \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > /dev/null 2>&1
  python scripts/ncu_summary.py report gpurun_out/r1d/prof_$tag.ncu-rep --json gpurun_out/r1d/ncu_full_$tag.json > gpurun_out/r1d/sum_$tag.txt 2>&1; echo "$tag done"; }
full k_win_wide_C5a k_win_wide 2 --config C5a --tuples-log2 26
full k_vh_build_tile_C5a k_vh_build_tile 2 --config C5a --tuples-log2 26
full k_win_block_C3_G64 k_win_block 4 --config C3 --groups 64 --tuples-log2 26
full k_pane_agg_C5a k_pane_agg 2 --config C5a --tuples-log2 26
