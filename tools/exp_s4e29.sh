OUT=gpurun_out/s4e29; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -k "reduce" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
