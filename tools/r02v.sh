set -u
OUT=gpurun_out/r02v; mkdir -p $OUT
timeout 900 python tools/ab_conv.py base noop base noop > $OUT/ab_conv.txt 2>&1
python tools/copy_floor.py > $OUT/copy_floor.txt 2>&1
