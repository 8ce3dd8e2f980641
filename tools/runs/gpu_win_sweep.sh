#!/bin/bash
# window-kernel configuration sweep + CUDA-graph experiment: bash tools/gpu_win_sweep.sh TAG
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
for c in C2 C3; do
  python tools/graph_exp.py $c > $OUT/${TAG}_graph_$c.json 2>&1
  for K in 1 2 3 4; do
    KRCV_WIN_K=$K timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_K$K.json 2>/dev/null
  done
  for NBC in 4 8 16 32 64; do
    KRCV_WIN_NBC=$NBC timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_nbc$NBC.json 2>/dev/null
  done
done
echo done
