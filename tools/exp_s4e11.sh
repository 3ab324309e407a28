OUT=gpurun_out/s4e11; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_probe.py > $OUT/memcheck.log 2>&1; echo "memcheck $?" >> $OUT/status.txt
timeout 1500 compute-sanitizer --tool racecheck --racecheck-report hazard --print-limit 20 python tools/sanitize_probe.py > $OUT/racecheck.log 2>&1; echo "racecheck $?" >> $OUT/status.txt
