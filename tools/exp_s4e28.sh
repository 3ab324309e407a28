OUT=gpurun_out/s4e28; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for cfg in 2:1 4:1 8:1; do LOP_CONV_CFG=$cfg timeout 300 python tools/tune_conv.py $cfg 2>&1 | grep sobel3x3_u8 >> $OUT/sobel_u8.txt; done
for ts in 4 8 16; do LOP_REDUCE_TS=$ts timeout 300 python bench.py --steps 5 --e2e-steps 0 --no-cpu-baseline 2>/dev/null | python -c "
import json,sys; d=json.load(sys.stdin); c=d['filters']['conv_4096']; print('ts=$ts', c['erode5x5_u8']['ms'], c['dilate3x3_f32']['ms'])" >> $OUT/reduce_ts.txt; done
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "reduce or conv_tile_configs" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
