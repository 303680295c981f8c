#!/usr/bin/env bash
# Build a variant of libtc_b200.so with extra nvcc defines into build_variant/NAME/ (A/B
# experiments: TC_B200_LIB=build_variant/NAME/libtc_b200.so python tools/ab_option.py ...).
#   bash tools/build_variant.sh NAME "-DTC_TS_L=2"
set -e
NAME=$1; shift
FLAGS="$*"
ROOT=$(cd "$(dirname "$0")/.." && pwd)
OUT=$ROOT/build_variant/$NAME
mkdir -p $OUT
NV="/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -ffp-contract=off --expt-relaxed-constexpr -I$ROOT/include $FLAGS"
PK=$ROOT/paper_conf_sigmod_hu0l21_b200/csrc
pids=""
for f in $PK/*.cu $PK/*.cpp; do
  b=$(basename $f); b=${b%.*}
  $NV -c $f -o $OUT/$b.o &
  pids="$pids $!"
done
for p in $pids; do wait $p; done
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared $OUT/*.o -o $OUT/libtc_b200.so -ldl
echo "built $OUT/libtc_b200.so"
