# §8(f) rows f1 and f2 on B200 (§6.3-6.4): every line is a
# clocked bench.py JSON line.  Output: gpurun_out/sweeps/*.jsonl
#   f1  CM2 (σ + int64 high-cardinality GROUP BY) and the SELECT_n predicate-cost sweep (Fig. 10a)
#   f2  task-size φ sweep (Figs. 12-13) device-resident and end-to-end, slide sweep (Fig. 11)
#       device-resident and end-to-end, SELECT10 slide sweep (selection is slide-insensitive,
#       L2044-2046), Fig. 13 window-independence runs (SELECT1 at ω(1,1), ω(1024,1), ω(1024,1024))
mkdir -p gpurun_out/sweeps
export PATH=/usr/local/cuda/bin:$PATH
run() { out=$1; shift; echo "== $*" >&2; timeout 500 python bench.py --no-cpu "$@" 2>>gpurun_out/sweeps/err.txt | tail -1 >> $out || true; }
o=gpurun_out/sweeps/f1_cm2.jsonl; : > $o
run $o --config CM2 --steps 5 --warmup 3
run $o --config CM2 --rate 4096 --steps 5 --warmup 3
o=gpurun_out/sweeps/f3_join.jsonl; : > $o
run $o --config JOIN --join-r 1 --steps 5 --warmup 3
run $o --config JOIN --join-r 4 --steps 5 --warmup 3
run $o --config JOIN --join-r 16 --steps 5 --warmup 3
o=gpurun_out/sweeps/f1_select_n.jsonl; : > $o
for n in 1 4 16 64; do run $o --config C2 --sel 0.5 --npred $n --steps 5 --warmup 3 --no-e2e; done
o=gpurun_out/sweeps/f2_task_size.jsonl; : > $o
for mb in 16 64 256 1024 2048 4096 8192; do run $o --config C3 --task-mb $mb --e2e-task-mb $(( mb < 1024 ? mb : 1024 )) --steps 5 --warmup 3; done
o=gpurun_out/sweeps/f2_slide.jsonl; : > $o
for l in 64 256 1024 4096 16384 32768; do run $o --config C3 --size 32768 --slide $l --steps 5 --warmup 3; done
o=gpurun_out/sweeps/f2_select10_slide.jsonl; : > $o
for l in 1 16 64 256 1024; do run $o --config C2 --npred 10 --size 1024 --slide $l --steps 5 --warmup 3 --no-e2e; done
o=gpurun_out/sweeps/f2_fig13_window_independence.jsonl; : > $o
run $o --config C2 --npred 1 --size 1 --slide 1 --steps 5 --warmup 3 --no-e2e
run $o --config C2 --npred 1 --size 1024 --slide 1 --steps 5 --warmup 3 --no-e2e
run $o --config C2 --npred 1 --size 1024 --slide 1024 --steps 5 --warmup 3 --no-e2e
for f in gpurun_out/sweeps/*.jsonl; do echo "# $f"; python scripts/bench_table.py $f; done
