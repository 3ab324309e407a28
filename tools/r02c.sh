set -u
OUT=gpurun_out/r02c; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.log 2>&1
timeout 600 python -m pytest tests/test_dist_gpu.py -q -p no:cacheprovider > $OUT/pytest_dist.log 2>&1; echo "dist $?" >> $OUT/status.txt
timeout 900 python tools/ab_variants.py np0 np1 np2 r128 > $OUT/ab.txt 2>&1; echo "ab $?" >> $OUT/status.txt
