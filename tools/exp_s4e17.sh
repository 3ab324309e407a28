OUT=gpurun_out/s4e17; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 600 python tools/pipe_frames_sweep.py 10 > $OUT/sweep.txt 2>&1
LOP_PIPELINE_BUFS=4 timeout 600 python tools/pipe_frames_sweep.py 10 >> $OUT/sweep.txt 2>&1
