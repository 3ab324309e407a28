set -u
OUT=gpurun_out/r02b; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 600 python -m pytest tests/test_dist_gpu.py -q -p no:cacheprovider > $OUT/pytest_dist.log 2>&1; echo "dist $?" >> $OUT/status.txt
timeout 300 ./tools/mio_probe > $OUT/mio_probe.txt 2>&1; echo "mio $?" >> $OUT/status.txt
timeout 900 python tools/sweep_bilateral.py all > $OUT/sweep_bilateral.jsonl 2> $OUT/sweep.err; echo "sweep $?" >> $OUT/status.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:bilateral_pair -s 3 -c 1 -o $OUT/prof_pair -f python bench.py --steps 5 --warmup 3 --no-extras --no-cpu-baseline --e2e-steps 0 --no-partitioned > $OUT/ncu_full.log 2>&1; echo "full $?" >> $OUT/status.txt
