# launch lists for the weak configs + a C3 bench line with clocks (1 GPU)
mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/bench_c3.log 2>&1; tail -1 gpurun_out/bench_c3.log | cut -c1-300
python -c "import json;d=json.loads(open('gpurun_out/bench_c3.log').read().strip().splitlines()[-1]);print(d['clocks'])"
CONFIGS="C3 --groups 64|C3 --groups 1024|C3 --groups 16384 --task-mb 128|C3 --groups 65536 --task-mb 64|C5a|C5b|C4 --rate 64|C2" LOG2=26 bash scripts/ncu_launches.sh
for f in gpurun_out/launches_*.csv; do echo "== $f"; python scripts/ncu_summary.py launches $f | head -12; done
