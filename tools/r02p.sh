set -u
OUT=gpurun_out/r02p; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke $?" >> $OUT/status.txt
timeout 1500 python -m pytest tests/test_bench_gpu.py -q -p no:cacheprovider -x > $OUT/pytest_bench.log 2>&1; echo "benchtests $?" >> $OUT/status.txt
