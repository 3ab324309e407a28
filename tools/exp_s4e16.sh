OUT=gpurun_out/s4e16; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "pipeline" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
timeout 900 python bench.py --no-extras --no-cpu-baseline > $OUT/bench.json 2> $OUT/bench.err; echo "bench $?" >> $OUT/status.txt
timeout 900 python bench.py --no-extras --no-cpu-baseline --e2e-steps 30 > $OUT/bench30.json 2> $OUT/bench30.err; echo "bench30 $?" >> $OUT/status.txt
