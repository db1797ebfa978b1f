# ncu --set full of chosen kernels on chosen configs (1 GPU); reports under gpurun_out/
mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
run() { tag=$1; kre=$2; shift 2
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$kre -s ${SKIP:-2} -c 1 -o gpurun_out/prof_$tag \
    python bench.py --steps 1 --warmup 1 --tuples-log2 ${LOG2:-26} --no-e2e --no-cpu "$@" > gpurun_out/ncu_$tag.log 2>&1
  echo "$tag rc=$?"; python scripts/ncu_summary.py report gpurun_out/prof_$tag.ncu-rep --json gpurun_out/prof_$tag.json | head -40; }
run c3g64_scan k_pane_cnt --config C3 --groups 64
run c3g64_win k_win_packed --config C3 --groups 64
run c3g1024_win k_win_fused --config C3 --groups 1024
