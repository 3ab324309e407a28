set -u
OUT=gpurun_out/r02f; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests/test_local_gpu.py tests/test_parity_gpu.py -q -p no:cacheprovider -k "local or chain" > $OUT/pytest.log 2>&1; echo "tests $?" >> $OUT/status.txt
timeout 300 python tools/time_local.py > $OUT/time_local.jsonl 2>&1; echo "time $?" >> $OUT/status.txt
LOP_LOCAL_SMALL=0 timeout 300 python tools/time_local.py > $OUT/time_local_nosmall.jsonl 2>&1
