OUT=gpurun_out/s4e15; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for cfg in 16:1 4:2 8:2 16:2; do for c in 1 2 3 4 6; do
  if [ $cfg = 16:1 ] && [ $c != 1 ]; then continue; fi
  r=$(LOP_CONV_CFG=$cfg LOP_CONV_CTAS_PER_SM=$c timeout 120 python tools/time_conv_u8.py 5 2>&1 | tail -1)
  echo "cfg=$cfg ctas_per_sm=$c $r" >> $OUT/sweep.txt
done; done
