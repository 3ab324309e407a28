set -u
OUT=gpurun_out/r02i; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
LOP_LOCAL_CFG=64:2 timeout 600 ncu --set full --clock-control none --import-source on -k regex:local_small -s 2 -c 1 -o $OUT/prof_local -f python tools/time_local.py > $OUT/ncu.log 2>&1
