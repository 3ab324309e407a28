OUT=gpurun_out/s4e19; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -k "signed_swar or config3 or conv_small" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
timeout 300 python tools/tune_chain.py 8 > $OUT/chain.jsonl 2>&1
