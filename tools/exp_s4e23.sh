OUT=gpurun_out/s4e23; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -k "bilateral" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
timeout 300 python tools/tune_bilateral.py 0:1 0:1:m > $OUT/tune.jsonl 2>&1
LOP_BILATERAL_FACTOR=0 timeout 300 python tools/tune_bilateral.py 0:1:m > $OUT/tune_nofactor.jsonl 2>&1
