#!/bin/bash
# SM-local task regions for the window kernels (KRCV_WIN_SCHED=1 default) vs the global counter
TAG=${1:-r01ax}; OUT=gpurun_out; mkdir -p $OUT
for c in C2 C3 C5 C4; do
  for S in 0 1; do
    KRCV_WIN_SCHED=$S timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_S$S.json 2> $OUT/${TAG}_bench_${c}_S$S.err
  done
done
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_window_variants.py -x -q > $OUT/${TAG}_pytest.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest.log
timeout 900 ncu --set full --clock-control none --import-source on -k regex:window_kernel -s 2 -c 1 \
    -o $OUT/${TAG}_window_C2 -f python bench.py --steps 1 --warmup 2 --no-cpu-baseline --no-alt > $OUT/${TAG}_ncu_full.log 2>&1
echo done
