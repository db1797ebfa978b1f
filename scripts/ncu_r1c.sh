# session 3: overlap parity test + ncu --set full (source) of the window kernels and the C5a scan
mkdir -p gpurun_out/r1c
export PATH=/usr/local/cuda/bin:$PATH
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k overlap > gpurun_out/r1c/t_ovl.log 2>&1; echo "ovl_rc=$?"; tail -2 gpurun_out/r1c/t_ovl.log
full() { tag=$1; kre=$2; skip=$3; shift 3
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$kre -s $skip -c 1 -o gpurun_out/r1c/prof_$tag \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > /dev/null 2>&1
  python scripts/ncu_summary.py report gpurun_out/r1c/prof_$tag.ncu-rep --json gpurun_out/r1c/ncu_full_$tag.json | head -12; }
full k_win_block_C3_G64 k_win_block 9 --config C3 --groups 64 --tuples-log2 26
full k_vh_build_cta_C5a k_vh_build_cta 3 --config C5a --tuples-log2 26
full k_win_fused_C5a k_win_fused 3 --config C5a --tuples-log2 26
full k_pane_agg_C5a k_pane_agg 3 --config C5a --tuples-log2 26
full k_pane_agg_C5b k_pane_agg 3 --config C5b --tuples-log2 26
ls gpurun_out/r1c
