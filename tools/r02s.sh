set -u
OUT=gpurun_out/r02s; mkdir -p $OUT
timeout 600 ncu --set full --clock-control none --import-source on -k regex:local_small -s 2 -c 1 -o $OUT/prof_local -f python tools/time_local.py > $OUT/ncu.log 2>&1
