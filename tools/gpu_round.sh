#!/bin/bash
# One GPU session: build check, smoke, GPU tests, bench, ncu launch list + one
# full capture of the top kernel.  Usage (from the repo root, under gpurun):
#   tools/gpu_round.sh [tag] [what...]    what in: smoke tests bench ncu full peaks
set -u
TAG=${1:-r01}
shift || true
WHAT=${*:-"smoke tests bench ncu full"}
OUT=gpurun_out/$TAG
mkdir -p "$OUT"
nvidia-smi > "$OUT/nvidia-smi.txt" 2>&1
nproc > "$OUT/nproc.txt"
python -c "import __graft_entry__ as g; g.build()" > "$OUT/build.log" 2>&1
for w in $WHAT; do
  case $w in
    smoke)
      timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > "$OUT/smoke.log" 2>&1
      echo "smoke exit $?" >> "$OUT/status.txt" ;;
    tests)
      timeout 1800 python -m pytest tests -m gpu -q -p no:cacheprovider --timeout=900 \
        > "$OUT/pytest_gpu.log" 2>&1
      echo "tests exit $?" >> "$OUT/status.txt" ;;
    bench)
      timeout 900 python bench.py > "$OUT/bench.json" 2> "$OUT/bench.err"
      echo "bench exit $?" >> "$OUT/status.txt" ;;
    reference)
      timeout 600 python bench.py --impl reference --steps 3 --warmup 1 \
        > "$OUT/bench_reference.json" 2> "$OUT/bench_reference.err"
      echo "bench_reference exit $?" >> "$OUT/status.txt" ;;
    peaks)
      timeout 300 ./tools/peaks > "$OUT/peaks.txt" 2>&1
      echo "peaks exit $?" >> "$OUT/status.txt" ;;
    ncu)
      timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"bilateral|conv|local" -c 60 --csv \
        --log-file "$OUT/launches.csv" python bench.py --steps 20 --warmup 3 --no-extras \
        --no-cpu-baseline --e2e-steps 0 --no-partitioned > "$OUT/ncu_launch_bench.log" 2>&1
      echo "ncu exit $?" >> "$OUT/status.txt" ;;
    full)
      timeout 900 ncu --set full --clock-control none --import-source on \
        -k regex:bilateral_ -s 3 -c 1 -o "$OUT/prof_bilateral" -f \
        python bench.py --steps 5 --warmup 3 --no-extras --no-cpu-baseline --e2e-steps 0 --no-partitioned \
        > "$OUT/ncu_full.log" 2>&1
      echo "full exit $?" >> "$OUT/status.txt" ;;
    fullconv)
      timeout 900 ncu --set full --clock-control none --import-source on \
        -k regex:conv -s 2 -c 4 -o "$OUT/prof_conv" -f \
        python tools/conv_probe.py > "$OUT/ncu_fullconv.log" 2>&1
      echo "fullconv exit $?" >> "$OUT/status.txt" ;;
  esac
done
ls -la "$OUT" > "$OUT/listing.txt"
