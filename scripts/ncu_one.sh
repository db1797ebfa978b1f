# usage: KRE=<kernel regex> SKIP=n TAG=name ARGS="bench args" bash scripts/ncu_one.sh
mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 600 ncu --set full --clock-control none --import-source on -k regex:$KRE -s ${SKIP:-3} -c 1 -o gpurun_out/prof_$TAG \
    python bench.py --steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu $ARGS > /dev/null 2>&1
python scripts/ncu_summary.py report gpurun_out/prof_$TAG.ncu-rep | head -30
