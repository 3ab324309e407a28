OUT=gpurun_out/s4e22; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "conv or config3 or swar or tile_configs" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
for sp in 1 0; do for cfg in 8:1 16:1 4:1; do
LOP_CONV_SPLIT=$sp LOP_CONV_CFG=$cfg timeout 300 python tools/tune_conv.py $cfg 2>&1 | sed "s/^/split=$sp /" >> $OUT/sweep.txt
done; done
