# end-of-session evidence for the default bench line: the bench JSON (with e2e,
# cpu baseline, clocks), the ncu launch list of the same command, and ncu --set full
# of the dominant kernels at the bench's launch configuration
mkdir -p gpurun_out/fin; rm -f gpurun_out/fin/*
export PATH=/usr/local/cuda/bin:$PATH
timeout 600 python bench.py > gpurun_out/fin/bench_default.jsonl 2> gpurun_out/fin/bench_default.err; echo bench_rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/fin/launches_default.csv \
   python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo launches_rc=$?
python scripts/ncu_summary.py launches gpurun_out/fin/launches_default.csv > gpurun_out/fin/launches_default.txt
gzip -f gpurun_out/fin/launches_default.csv
full() { tag=$1; kre=$2; skip=$3; shift 3
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$kre -s $skip -c 1 -o gpurun_out/fin/prof_$tag \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > /dev/null 2>&1
  python scripts/ncu_summary.py report gpurun_out/fin/prof_$tag.ncu-rep --json gpurun_out/fin/ncu_full_$tag.json > gpurun_out/fin/sum_$tag.txt 2>&1
  rm -f gpurun_out/fin/prof_$tag.ncu-rep; echo "$tag done"; }
full k_pane_cnt_C3_G64 k_pane_cnt 2 --config C3 --groups 64
full k_win_block_C3_G64 k_win_block 3 --config C3 --groups 64
full k_win_wide_C5a k_win_wide 4 --config C5a --task-mb 1024 --tuples-log2 26
full k_pane_agg_C5a k_pane_agg 2 --config C5a --task-mb 1024 --tuples-log2 26
bash scripts/bench_all.sh > /dev/null 2>&1; cp gpurun_out/bench_all.jsonl gpurun_out/fin/bench_all.jsonl
ls gpurun_out/fin
