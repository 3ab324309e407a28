OUT=gpurun_out/s4e13; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
./tools/ffma2_probe > $OUT/ffma2_probe.txt 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "convolve2 or sobel_magnitude or reduce" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
