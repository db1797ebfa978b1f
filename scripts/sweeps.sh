# §8(f) f2: the paper's task-size (Figs. 12-13) and slide (Fig. 11) sweeps on B200,
# device-resident, C3 G=64 (Syn, AVG GROUP BY, count window).  Output: gpurun_out/sweeps/*.jsonl
mkdir -p gpurun_out/sweeps
export PATH=/usr/local/cuda/bin:$PATH
t=gpurun_out/sweeps/task_size.jsonl; : > $t
for tm in 16 64 256 1024 2048 4096 8192; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --config C3 --task-mb $tm 2>/dev/null | tail -1 >> $t
done
s=gpurun_out/sweeps/slide.jsonl; : > $s
for sl in 64 256 1024 4096 16384 32768; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --config C3 --slide $sl 2>/dev/null | tail -1 >> $s
done
for sl in 1 10 60; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --config C4 --rate 4096 --slide $sl 2>/dev/null | tail -1 >> $s
done
python - <<'PY'
import json
for f in ("task_size", "slide"):
    print("==", f)
    for l in open(f"gpurun_out/sweeps/{f}.jsonl"):
        try: d = json.loads(l)
        except Exception: continue
        r = d["roofline"]
        print(f'{d["config"]["workload"][:90]:90s} phi={d["config"]["task_bytes"]>>20:5d}MiB {d["value"]:.3e} t/s {d["input_gbs"]:7.1f} GB/s ms={d["ms_per_step"]:.3f} scan_frac={r["frac"] and round(r["frac"],3)} windows={d["config"]["windows_per_step"]}')
PY
