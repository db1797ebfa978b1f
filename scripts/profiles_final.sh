# Round-end evidence (profiles/r02): GPU test suite + smoke, the default bench line (e2e + oracle
# baseline + clocks), every config device-resident with clocks, e2e lines, the ncu launch list of the
# default command, ncu --set full summaries of the dominant kernels at the bench's launch
# configuration, the live kernel timeline of a default step, and the read-bandwidth microbenchmark.
set -x
O=gpurun_out/fin; mkdir -p $O; rm -f $O/*
export PATH=/usr/local/cuda/bin:$PATH
timeout 2400 python -m pytest tests -m gpu -q > $O/gpu_tests.log 2>&1; echo tests_rc=$?
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke_rc=$?
timeout 900 python bench.py > $O/bench_default.jsonl 2> $O/bench_default.err; echo bench_rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_default.csv \
   python bench.py --steps 2 --warmup 1 --no-e2e --no-cpu > /dev/null 2>&1; echo launches_rc=$?
python scripts/ncu_summary.py launches $O/launches_default.csv > $O/launches_default.txt
gzip -f $O/launches_default.csv
python scripts/trace_step.py > $O/trace_default.txt 2>&1
full() { tag=$1; kre=$2; skip=$3; shift 3
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$kre -s $skip -c 1 -o $O/prof_$tag \
    python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > /dev/null 2>&1
  python scripts/ncu_summary.py report $O/prof_$tag.ncu-rep --json $O/ncu_full_$tag.json > $O/sum_$tag.txt 2>&1
  python scripts/ncu_lines.py $O/prof_$tag.ncu-rep 25 > $O/lines_$tag.txt 2>&1
  rm -f $O/prof_$tag.ncu-rep; echo "$tag done"; }
full k_pane_cnt_C3_G64 k_pane_cnt 2 --config C3 --groups 64
full k_win_block_reg_C3_G64 k_win_block_reg 3 --config C3 --groups 64
full k_wb_rows_C3_G64 k_wb_rows 3 --config C3 --groups 64
full k_pane_agg_C5a k_pane_agg 2 --config C5a
full k_select_C2 k_select 0 --config C2
full k_win_block_reg_C3_G256 k_win_block_reg 3 --config C3 --groups 256
full k_bkt_rows_C3_G1024 k_bkt_rows 2 --config C3 --groups 1024
bash scripts/bench_all.sh $O/bench_all_configs.jsonl > $O/bench_all_configs.txt 2>&1
for c in C1 C2 C4 C5a C5b SG1; do timeout 600 python bench.py --no-cpu --steps 3 --warmup 3 --config $c 2>>$O/e2e.err | tail -1; done > $O/bench_e2e_configs.jsonl
./build_var/ubr > $O/ubench_read_bw.txt 2>&1
mkdir -p gpurun_out/sweeps; bash scripts/sweeps.sh > gpurun_out/sweeps/tables.txt 2>&1
ls $O
