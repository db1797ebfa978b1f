mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
for k in k_bkt_emit k_bkt_count; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s 3 -c 1 -o gpurun_out/prof_$k \
    python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu --config C3 --groups 65536 --task-mb 256 > /dev/null 2>&1
python scripts/ncu_summary.py report gpurun_out/prof_$k.ncu-rep | head -30
done
