set -u
OUT=gpurun_out/r02g; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
LOP_DEBUG_SELECT=1 timeout 300 python tools/time_local.py > $OUT/time_local.jsonl 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:local_small -s 2 -c 1 -o $OUT/prof_local -f python tools/time_local.py > $OUT/ncu.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_sep_kernel -s 2 -c 1 -o $OUT/prof_u8g -f python tools/conv_probe_u8.py > $OUT/ncu_u8.log 2>&1
