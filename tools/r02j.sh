set -u
OUT=gpurun_out/r02t; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 300 python -m pytest tests/test_local_gpu.py -q -p no:cacheprovider -x > $OUT/pytest_local.log 2>&1; echo "local $?" >> $OUT/status.txt
timeout 900 python tools/sweep_local.py > $OUT/sweep_local.jsonl 2> $OUT/sweep_local.err
LOP_DEBUG_SELECT=1 timeout 300 python tools/time_local.py > $OUT/time_local.jsonl 2>&1
