#!/bin/bash
# register-cap variants of the window kernels: bash tools/gpu_mb.sh TAG
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
for lib in libkrcv.so libkrcv_mb7.so libkrcv_mb8.so; do
  for c in C2 C3 C4; do
    KRCV_LIB=$lib timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_${lib%.so}.json 2> /dev/null
  done
  KRCV_LIB=$lib KRCV_CHUNK=4 timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_C2_chunk4_${lib%.so}.json 2> /dev/null
done
echo done
