set -u
OUT=gpurun_out/r02l; mkdir -p $OUT
timeout 900 python tools/ab_conv.py base sus1k sus20k base sus1k sus20k > $OUT/ab_conv.txt 2>&1
timeout 600 python tools/ab_variants.py base sus1k > $OUT/ab_pair.txt 2>&1
