mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "bucket or c3_groupby" > gpurun_out/t_bucket.log 2>&1
echo "tests_rc=$?"; tail -3 gpurun_out/t_bucket.log
for a in "--groups 16384 --task-mb 512" "--groups 65536 --task-mb 256"; do
timeout 300 python bench.py --config C3 $a --steps 3 --warmup 2 --no-cpu --no-e2e 2>&1 | tail -2 | cut -c1-200
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_bkt_emit -s 3 -c 1 -o gpurun_out/prof_k_bkt_emit \
    python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu --config C3 --groups 65536 --task-mb 256 > /dev/null 2>&1
python scripts/ncu_summary.py report gpurun_out/prof_k_bkt_emit.ncu-rep | head -30
