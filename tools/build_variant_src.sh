#!/bin/bash
# Build liblop.so from another source tree (e.g. `git archive <rev>` of csrc/ and
# include/) for A/B against the working tree:
#   tools/build_variant_src.sh <name> <tree-root> [nvcc defines...]
# -> build/variants/liblop_<name>.so  (select with LOP_LIBRARY=...)
set -e
NAME=$1; SRC=$2; shift 2
ROOT=$(cd "$(dirname "$0")/.." && pwd)
PKG=$SRC/paper_conf_ipps_membarthhtke12_b200
OUT=$ROOT/build/variants/$NAME
mkdir -p "$OUT"
objs=()
for src in "$PKG"/csrc/*.cu "$PKG"/csrc/*.cpp; do
  o=$OUT/$(basename "${src%.*}").o
  extra=()
  [[ $src == *.cu ]] && extra=(-Xptxas -v --expt-relaxed-constexpr)
  nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -lineinfo -Xcompiler -fPIC "${extra[@]}" \
    -I "$SRC/include" -I "$PKG/csrc" "$@" -c "$src" -o "$o" 2> "$o.log" &
  objs+=("$o")
done
wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -cudart static -o "$ROOT/build/variants/liblop_$NAME.so" "${objs[@]}"
