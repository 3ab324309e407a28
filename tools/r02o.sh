set -u
OUT=gpurun_out/r02o; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 compute-sanitizer --tool memcheck --print-limit 20 python tools/sanitize_local.py > $OUT/memcheck.log 2>&1; echo "memcheck $?" >> $OUT/status.txt
timeout 1200 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_local.py > $OUT/racecheck.log 2>&1; echo "racecheck $?" >> $OUT/status.txt
timeout 1200 compute-sanitizer --tool initcheck --print-limit 20 python tools/sanitize_local.py > $OUT/initcheck.log 2>&1; echo "initcheck $?" >> $OUT/status.txt
