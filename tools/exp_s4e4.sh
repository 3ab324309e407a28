set -u
OUT=gpurun_out/s4e4; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider -x -k "chain" > $OUT/pytest_chain.log 2>&1; echo "pytest_chain $?" >> $OUT/status.txt
timeout 300 python tools/tune_chain.py 8 > $OUT/chain_stream.jsonl 2>&1
for r in 12 16 24; do LOP_CHAIN_ROWS=$r timeout 300 python tools/tune_chain.py 8 2>&1 | grep fused | sed "s/^/rows=$r /" >> $OUT/chain_rows.txt; done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:chain_stream -s 2 -c 2 -o $OUT/prof_chain -f python tools/tune_chain.py 8 > $OUT/ncu.log 2>&1; echo "ncu $?" >> $OUT/status.txt
