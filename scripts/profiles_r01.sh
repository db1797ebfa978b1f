# round-1 evidence: launch list of the default bench command, ncu --set full of the
# dominant kernels, the default bench line (with e2e + cpu baseline), all configs
mkdir -p gpurun_out/r01
export PATH=/usr/local/cuda/bin:$PATH
timeout 600 python bench.py > gpurun_out/r01/bench_default.jsonl 2> gpurun_out/r01/bench_default.err; echo bench_rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/r01/launches_default.csv \
   python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo launches_rc=$?
python scripts/ncu_summary.py launches gpurun_out/r01/launches_default.csv > gpurun_out/r01/launches_default.txt
full() { tag=$1; kre=$2; skip=$3; shift 3
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$kre -s $skip -c 1 -o gpurun_out/r01/prof_$tag \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > /dev/null 2>&1
  python scripts/ncu_summary.py report gpurun_out/r01/prof_$tag.ncu-rep --json gpurun_out/r01/ncu_full_$tag.json > /dev/null; echo "$tag done"; }
full k_pane_cnt_C3_G64 k_pane_cnt 9 --config C3 --groups 64
full k_win_block_C3_G64 k_win_block 9 --config C3 --groups 64
full k_bkt_emit_C3_G65536 k_bkt_emit 33 --config C3 --groups 65536 --task-mb 256
full k_pane_bucket_C3_G65536 k_pane_bucket 33 --config C3 --groups 65536 --task-mb 256
full k_select_C2 k_select 2 --config C2
bash scripts/bench_all.sh > /dev/null 2>&1; cp gpurun_out/bench_all.jsonl gpurun_out/r01/bench_all_configs_device_resident.jsonl
ls gpurun_out/r01
