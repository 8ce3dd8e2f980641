#!/bin/bash
# window_kernel_blk (KRCV_WIN_K=9/10): variant tests, parity, A/B bench
TAG=${1:-r01at}; OUT=gpurun_out; mkdir -p $OUT
timeout 600 python -m pytest tests/test_gpu_window_variants.py -x -q -k blk > $OUT/${TAG}_pytest_variants.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_variants.log
for c in C2 C3 C5 C4; do
  for K in 0 9 10; do
    if [ $K = 0 ]; then unset KRCV_WIN_K; else export KRCV_WIN_K=$K; fi
    timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_K$K.json 2> $OUT/${TAG}_bench_${c}_K$K.err
  done
done
unset KRCV_WIN_K
for K in 9 10; do
  KRCV_WIN_K=$K timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_property.py -x -q > $OUT/${TAG}_pytest_K$K.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_K$K.log
done
echo done
