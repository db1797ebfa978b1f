# device-resident bench line for every config (exploration; not the driver's bench)
mkdir -p gpurun_out
out=gpurun_out/bench_all.jsonl; : > $out
run() { echo "== $*" >&2; timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e "$@" 2>gpurun_out/bench_err.txt | tail -1 >> $out || true; tail -2 gpurun_out/bench_err.txt >&2; }
run --config C1 --task-mb 32
run --config C2 --sel 0.5 --task-mb 1024
run --config C2 --sel 0.1 --task-mb 1024
run --config C2 --sel 1.0 --task-mb 1024
run --config C3 --groups 64 --task-mb 4096
run --config C3 --groups 256 --task-mb 1024
run --config C3 --groups 4096 --task-mb 1024
run --config C3 --groups 1024 --task-mb 1024
run --config C3 --groups 16384 --task-mb 512
run --config C3 --groups 65536 --task-mb 256
run --config C4 --rate 64 --task-mb 4096
run --config C4 --rate 4096 --task-mb 4096
run --config C5a --task-mb 4096
run --config C5b --task-mb 4096
run --config SG1 --task-mb 4096
python - <<'PY'
import json
for l in open("gpurun_out/bench_all.jsonl"):
    try: d=json.loads(l)
    except Exception: continue
    r=d["roofline"]
    print(f'{d["config"]["workload"][:60]:60s} {d["value"]:.3e} t/s {d["input_gbs"]:7.1f} GB/s  ms={d["ms_per_step"]:.2f} scan={r["achieved"] and round(r["achieved"])} GB/s frac={r["frac"] and round(r["frac"],3)} share={r["share_of_step"] and round(r["share_of_step"],2)} kern={r["kernel"]}/{r["window_kernels"]} rows={d["config"]["rows_per_step"]} tuples_out={d["config"]["out_tuples_per_step"]}')
PY
