OUT=gpurun_out/s4e5; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
for m in clamp constant; do for w in f32 u8; do
timeout 300 compute-sanitizer --tool memcheck --print-limit 5 python tools/chain_dbg.py $m $w > $OUT/san_${m}_$w.log 2>&1
done; done
