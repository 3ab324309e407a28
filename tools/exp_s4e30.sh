OUT=gpurun_out/s4e30; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "swar or config3 or conv_small or conv_tile" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
for i in 1 2; do
timeout 120 python tools/time_conv_u8.py 5 > $OUT/bin5_$i.json 2>&1
LOP_CONV_SWAR=7 timeout 120 python tools/time_conv_u8.py 5 > $OUT/sym_$i.json 2>&1
done
