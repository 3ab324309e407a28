OUT=gpurun_out/s4e6; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
CONST=0.5 timeout 300 python tools/time_modes.py > $OUT/modes_c05.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,smsp__inst_executed.sum,sm__inst_executed_pipe_xu.sum,smsp__cycles_active.max,smsp__cycles_active.min,smsp__cycles_active.avg,sm__cycles_active.max,sm__cycles_active.avg,l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum,smsp__inst_executed_op_ldgsts.sum --clock-control none -k regex:bilateral_pair -c 4 --csv python tools/mode_probe.py clamp constant > $OUT/ncu_modes.csv 2>&1
