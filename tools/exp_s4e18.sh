OUT=gpurun_out/s4e18; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -k "conv or config3 or chain or sobel" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
timeout 300 python tools/tune_conv.py 8:1 > $OUT/conv_new.jsonl 2>&1
LOP_CONV_SWAR=0 timeout 300 python tools/tune_conv.py 8:1 > $OUT/conv_noswar.jsonl 2>&1
timeout 300 python tools/tune_chain.py 8 > $OUT/chain.jsonl 2>&1
