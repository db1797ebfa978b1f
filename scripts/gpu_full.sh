mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/t_all.log 2>&1
echo "tests_rc=$?"; tail -3 gpurun_out/t_all.log
bash scripts/gpu_quick.sh
