#!/bin/bash
# tests + a short bench on the GPU box; outputs under gpurun_out/
mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS} > gpurun_out/gpu_tests.log 2>&1
echo "tests_rc=$?"; grep -E "passed|failed|FAILED|Error" gpurun_out/gpu_tests.log | head -20
timeout 600 python bench.py --steps ${STEPS:-5} --warmup 3 --cpu-seconds ${CPUS:-3} ${BENCH_ARGS} > gpurun_out/bench.log 2>&1
echo "bench_rc=$?"; tail -c 2500 gpurun_out/bench.log
