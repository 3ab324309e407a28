OUT=gpurun_out/s4e21; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:global_partial -s 2 -c 2 -o $OUT/prof_global -f python tools/global_probe.py > $OUT/ncu.log 2>&1; echo "ncu $?" >> $OUT/status.txt
