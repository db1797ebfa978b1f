mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_win_packed|k_vh_build|k_zero" -s 9 -c 6 -o gpurun_out/prof_win64 \
    python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu --config C3 --groups 64 > /dev/null 2>&1
python scripts/ncu_summary.py report gpurun_out/prof_win64.ncu-rep | head -80
