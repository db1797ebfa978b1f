# ncu --set full of one kernel at the bench's launch configuration, report kept in gpurun_out/
# usage: bash scripts/ncu_full.sh <tag> <kernel-regex> <launch-skip> [bench args...]
tag=$1; kre=$2; skip=$3; shift 3
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/ncu
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$kre -s $skip -c 1 -o gpurun_out/ncu/$tag -f \
  python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu "$@" > gpurun_out/ncu/$tag.log 2>&1
python scripts/ncu_summary.py report gpurun_out/ncu/$tag.ncu-rep --json gpurun_out/ncu/$tag.json > gpurun_out/ncu/$tag.txt 2>&1
echo "$tag done"
