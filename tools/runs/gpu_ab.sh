#!/bin/bash
# A/B of the two algorithms on the GPU box: bash tools/gpu_ab.sh TAG "C2 C3 C5" [steps]
TAG=$1; CFGS=${2:-"C2 C3 C5"}; ST=${3:-10}
OUT=gpurun_out; mkdir -p $OUT
for c in $CFGS; do for a in sweep prefix; do
  timeout 600 python bench.py --config $c --algo $a --steps $ST --warmup 3 --no-cpu-baseline > $OUT/${TAG}_bench_${c}_${a}.json 2> $OUT/${TAG}_bench_${c}_${a}.err
done; done
echo done
