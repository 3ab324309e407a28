OUT=gpurun_out/s4e26; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for so in build/variants/liblop_*.so; do
  v=$(basename "$so" .so)
  for t in auto 43 60 86; do
    if [ "$t" = auto ]; then unset LOP_PAIR_ROWS; else export LOP_PAIR_ROWS=$t; fi
    r=$(LOP_LIBRARY=$PWD/$so timeout 120 python tools/tune_bilateral.py 0:1 2>&1 | tail -1)
    echo "$v T=$t $r" >> $OUT/ab.txt
  done
  unset LOP_PAIR_ROWS
done
