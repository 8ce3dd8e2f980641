#!/bin/bash
# ncu --set full captures of the window kernel at C3, C4, C5 (one launch each)
TAG=${1:-r01bq}; OUT=gpurun_out; mkdir -p $OUT
for c in C3 C5 C4; do
  timeout 1200 ncu --set full --clock-control none --import-source on -k regex:window_kernel -s 2 -c 1 \
    -o $OUT/${TAG}_window_$c -f python bench.py --config $c --steps 1 --warmup 2 --no-cpu-baseline --no-alt > $OUT/${TAG}_ncu_$c.log 2>&1
done
echo done
