set -u
OUT=gpurun_out/r02n; mkdir -p $OUT
timeout 600 python tools/ab_variants.py base r144 r144nw3 r136 base r144 > $OUT/ab_pair.txt 2>&1
python -c "
import sys; sys.path.insert(0,'.')
import bench, torch
for i in range(3): print('ceiling GB/s per direction', round(bench.measure_copy_ceiling(torch.device('cuda',0), 64<<20), 2))
" > $OUT/ceiling.txt 2>&1
