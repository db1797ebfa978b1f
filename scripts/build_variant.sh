# build libsaber.so with extra -D flags into build_var/<name>.so (tuning experiments)
# usage: bash scripts/build_variant.sh <name> -DSB_P1_STAGES=3 ...
set -e
name=$1; shift
ROOT=$(cd "$(dirname "$0")/.." && pwd)
CS=$ROOT/paper_conf_sigmod_koliousiswfwcp16_b200/csrc
OUT=$ROOT/build_var/$name; mkdir -p $OUT
pids=""
for f in $CS/*.cu; do
  /usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC \
    --expt-relaxed-constexpr -diag-suppress 550 "$@" -I $ROOT/include -c $f -o $OUT/$(basename $f .cu).o & pids="$pids $!"
done
for p in $pids; do wait $p; done
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared $OUT/*.o -o $ROOT/build_var/$name.so
rm -rf $OUT
echo built build_var/$name.so
