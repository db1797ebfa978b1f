mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x > gpurun_out/t_all.log 2>&1
echo "tests_rc=$?"; tail -3 gpurun_out/t_all.log
for a in "--groups 16384 --task-mb 512" "--groups 65536 --task-mb 256"; do
timeout 300 python bench.py --config C3 $a --steps 3 --warmup 2 --no-cpu --no-e2e 2>&1 | tail -2 | cut -c1-200
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_bkt_count -s 3 -c 1 -o gpurun_out/prof_k_bkt_count \
    python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu --config C3 --groups 65536 --task-mb 256 > /dev/null 2>&1
python scripts/ncu_summary.py report gpurun_out/prof_k_bkt_count.ncu-rep | head -30
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_bk64k.csv python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu --config C3 --groups 65536 --task-mb 256 > /dev/null 2>&1; python scripts/ncu_summary.py launches gpurun_out/launches_bk64k.csv > gpurun_out/l.txt; head -8 gpurun_out/l.txt
