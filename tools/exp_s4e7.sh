OUT=gpurun_out/s4e7; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 300 python tools/time_modes.py > $OUT/modes_c0.json 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "bilateral or roi or band or frames or config1 or config2 or offset" > $OUT/pytest_bil.log 2>&1; echo "pytest_bil $?" >> $OUT/status.txt
timeout 900 python bench.py > $OUT/bench.json 2> $OUT/bench.err; echo "bench $?" >> $OUT/status.txt
