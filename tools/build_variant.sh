#!/bin/bash
# Build a variant of liblop.so with extra nvcc defines (kernel-config A/B):
#   tools/build_variant.sh <name> -DLOP_PAIR_NW=4 -DLOP_PAIR_MAXREG=168
# -> build/variants/liblop_<name>.so  (select with LOP_LIBRARY=...)
set -e
NAME=$1; shift
ROOT=$(cd "$(dirname "$0")/.." && pwd)
PKG=$ROOT/paper_conf_ipps_membarthhtke12_b200
OUT=$ROOT/build/variants/$NAME
mkdir -p "$OUT"
objs=()
for src in "$PKG"/csrc/*.cu "$PKG"/csrc/*.cpp; do
  o=$OUT/$(basename "${src%.*}").o
  extra=()
  [[ $src == *.cu ]] && extra=(-Xptxas -v --expt-relaxed-constexpr)
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC "${extra[@]}" \
    -I "$ROOT/include" -I "$PKG/csrc" "$@" -c "$src" -o "$o" 2> "$o.log" &
  objs+=("$o")
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o "$ROOT/build/variants/liblop_$NAME.so" "${objs[@]}"
grep -A3 "pair_kernelILi6" "$OUT/bilateral.o.log" | grep -E "Used|spill" || true
