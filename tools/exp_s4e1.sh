set -u
OUT=gpurun_out/s4e1; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "conv or config1 or small_shapes or bilateral_generic_and_tiled or roi" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
H=$PWD/build/variants/liblop_head.so
for size in 5 3; do
  LOP_LIBRARY=$H timeout 120 python tools/time_conv_u8.py $size > $OUT/u8_head_$size.json 2>&1
  timeout 120 python tools/time_conv_u8.py $size > $OUT/u8_new_$size.json 2>&1
  LOP_CONV_SWAR=1 timeout 120 python tools/time_conv_u8.py $size > $OUT/u8_plain_$size.json 2>&1
done
LOP_LIBRARY=$H timeout 300 python tools/time_small_bilateral.py > $OUT/small_head.json 2>&1
timeout 300 python tools/time_small_bilateral.py > $OUT/small_new.json 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:conv_sep -s 8 -c 1 -o $OUT/prof_u8 -f python tools/time_conv_u8.py 5 > $OUT/ncu.log 2>&1; echo "ncu $?" >> $OUT/status.txt
