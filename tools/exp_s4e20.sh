OUT=gpurun_out/s4e20; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "global" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
timeout 900 python bench.py --steps 20 --e2e-steps 0 --no-cpu-baseline > $OUT/bench.json 2> $OUT/bench.err; echo "bench $?" >> $OUT/status.txt
