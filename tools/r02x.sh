set -u
OUT=gpurun_out/r02x; mkdir -p $OUT
LOP_CONV_STREAM=1 timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_u8_stream -s 2 -c 1 -o $OUT/prof_stream -f python tools/conv_probe_u8.py > $OUT/ncu.log 2>&1
