set -u
OUT=gpurun_out/r02w; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 600 python tools/stream_check.py > $OUT/stream_check.txt 2>&1
for T in 16 24 32 48 64; do echo "T=$T"; LOP_STREAM_T=$T timeout 300 python tools/stream_check.py 2>&1 | tail -4; done > $OUT/stream_T.txt 2>&1
