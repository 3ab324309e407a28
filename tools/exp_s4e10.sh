OUT=gpurun_out/s4e10; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
H=$PWD/build/variants/liblop_head.so
for cfg in 8:1 16:1 4:1; do
LOP_CONV_CFG=$cfg LOP_LIBRARY=$H timeout 300 python tools/tune_conv.py $cfg > $OUT/conv_head_$cfg.jsonl 2>&1
LOP_CONV_CFG=$cfg timeout 300 python tools/tune_conv.py $cfg > $OUT/conv_new_$cfg.jsonl 2>&1
done
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "conv or chain or config3" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
