OUT=gpurun_out/s4e27; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -q -p no:cacheprovider -k "bilateral or band or frames or roi or offset or pipeline" > $OUT/pytest.log 2>&1; echo "pytest $?" >> $OUT/status.txt
timeout 300 python tools/time_modes.py > $OUT/modes.json 2>&1
timeout 300 python tools/tune_bilateral.py 0:1 > $OUT/tune.jsonl 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,smsp__inst_executed.sum --clock-control none -k regex:bilateral_pair -c 2 --csv python tools/mode_probe.py clamp > $OUT/ncu.csv 2>&1
