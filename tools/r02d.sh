set -u
OUT=gpurun_out/r02d; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_local_gpu.py -q -p no:cacheprovider -x > $OUT/pytest_local.log 2>&1; echo "local $?" >> $OUT/status.txt
