# launch list (device time per kernel) for a few configs; 1 GPU
# usage: CONFIGS="C3|C4 --rate 64" bash scripts/ncu_launches.sh
mkdir -p gpurun_out
export PATH=/usr/local/cuda/bin:$PATH
IFS='|' read -ra CFGS <<< "${CONFIGS:-C3 --groups 1024|C5b|C4 --rate 64|C2}"
for cfg in "${CFGS[@]}"; do
  tag=$(echo $cfg | tr -d ' -')
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$tag.csv \
     python bench.py --steps 1 --warmup 1 --tuples-log2 ${LOG2:-26} --no-e2e --no-cpu --config $cfg > /dev/null 2>&1
  echo "$tag rc=$?"
done
