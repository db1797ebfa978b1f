mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 600 python bench.py > gpurun_out/bench_default.jsonl 2> gpurun_out/bench_default.err; echo bench_rc=$?
tail -1 gpurun_out/bench_default.jsonl | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps({k: d[k] for k in ('value','ms_per_step','roofline','e2e','cpu_baseline','clocks','gpu_launches')})[:1500])"
bash scripts/sweeps.sh
