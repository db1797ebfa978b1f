# launch list + full profile of the scan kernel and the window kernels (1 GPU)
mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
TAG=${TAG:-q}
ARGS="--steps 1 --warmup 1 --tuples-log2 26 --no-e2e --no-cpu ${BENCH_ARGS}"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}.csv python bench.py $ARGS > /dev/null 2>&1
echo launches_rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:${KREGEX:-k_pane_agg} -s ${SKIP:-4} -c ${COUNT:-1} -o gpurun_out/prof_${TAG} python bench.py $ARGS > /dev/null 2>&1
echo full_rc=$?
