set -u
OUT=gpurun_out/r02u; mkdir -p $OUT
timeout 900 python tools/ab_conv.py base roll base roll > $OUT/ab_conv.txt 2>&1
