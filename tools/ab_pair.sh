#!/bin/bash
# A/B the pair-kernel build variants (build/variants/liblop_*.so) on 4096^2 13x13:
# auto T and a few fixed T per variant.  Run under gpurun.
OUT=${1:-gpurun_out/ab_pair}; mkdir -p "$OUT"
for so in build/variants/liblop_*.so; do
  v=$(basename "$so" .so)
  for t in auto 43 64 86 128; do
    if [ "$t" = auto ]; then unset LOP_PAIR_ROWS; else export LOP_PAIR_ROWS=$t; fi
    r=$(LOP_LIBRARY=$PWD/$so timeout 120 python tools/tune_bilateral.py 0:1 2>&1 | tail -1)
    echo "$v T=$t $r"
  done
  unset LOP_PAIR_ROWS
done > "$OUT/ab.txt" 2>&1
