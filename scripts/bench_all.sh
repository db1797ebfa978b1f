# device-resident bench line for every config (clocks sampled), one JSON line each;
# usage: bash scripts/bench_all.sh <out.jsonl> [extra bench args]
out=${1:-gpurun_out/bench_all.jsonl}; shift || true
mkdir -p $(dirname $out); : > $out
run() { echo "== $*" >&2; timeout 400 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e "$@" 2>>${out%.jsonl}.err | tail -1 >> $out || true; }
run --config C1 "$@"
run --config C2 --sel 0.5 "$@"
run --config C2 --sel 0.1 "$@"
run --config C2 --sel 1.0 "$@"
run --config C3 --groups 64 "$@"
run --config C3 --groups 256 "$@"
run --config C3 --groups 1024 "$@"
run --config C3 --groups 4096 "$@"
run --config C3 --groups 16384 "$@"
run --config C3 --groups 65536 "$@"
run --config C4 --rate 64 "$@"
run --config C4 --rate 4096 "$@"
run --config C5a "$@"
run --config C5b "$@"
run --config SG1 "$@"
run --config CM2 "$@"
python scripts/bench_table.py $out
