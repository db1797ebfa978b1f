# round-1 (session 3) evidence: launch list of the default bench command and
# ncu --set full captures of the dominant kernels at the bench's launch configuration
mkdir -p gpurun_out/r01b; rm -f gpurun_out/r01b/*
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01b/launches_default.csv \
   python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo launches_rc=$?
python scripts/ncu_summary.py launches gpurun_out/r01b/launches_default.csv > gpurun_out/r01b/launches_default.txt
full() { tag=$1; kre=$2; skip=$3; shift 3
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$kre -s $skip -c 1 -o gpurun_out/r01b/prof_$tag \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > /dev/null 2>&1
  python scripts/ncu_summary.py report gpurun_out/r01b/prof_$tag.ncu-rep --json gpurun_out/r01b/ncu_full_$tag.json > gpurun_out/r01b/sum_$tag.txt 2>&1
  ncu -i gpurun_out/r01b/prof_$tag.ncu-rep --page source --csv --print-source sass > gpurun_out/r01b/sass_$tag.csv 2>/dev/null
  gzip -f gpurun_out/r01b/sass_$tag.csv; rm -f gpurun_out/r01b/prof_$tag.ncu-rep; echo "$tag done"; }
full k_pane_cnt_C3_G64 k_pane_cnt 2 --config C3 --groups 64
full k_win_block_C3_G64 k_win_block 3 --config C3 --groups 64
full k_pane_agg_C5a k_pane_agg 2 --config C5a --task-mb 1024 --tuples-log2 26
full k_win_wide_C5a k_win_wide 4 --config C5a --task-mb 1024 --tuples-log2 26
full k_vh_build_tile_C5a k_vh_build_tile 4 --config C5a --task-mb 1024 --tuples-log2 26
full k_select_C2 k_select 3 --config C2 --task-mb 512
full k_bkt_emit_C3_G65536 k_bkt_emit 33 --config C3 --groups 65536 --task-mb 256
gzip -f gpurun_out/r01b/launches_default.csv; du -sh gpurun_out; ls gpurun_out/r01b
