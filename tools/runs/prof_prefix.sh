#!/bin/bash
# ncu evidence for the window-prefix path: bash tools/prof_prefix.sh TAG "C2 C3"
TAG=$1; CFGS=${2:-"C2 C3"}
OUT=gpurun_out; mkdir -p $OUT
for c in $CFGS; do
  timeout 600 python bench.py --config $c --algo prefix --steps 10 --warmup 3 --no-cpu-baseline > $OUT/${TAG}_bench_${c}_prefix.json 2> $OUT/${TAG}_bench_${c}_prefix.err
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/${TAG}_launches_${c}.csv \
      python bench.py --config $c --algo prefix --steps 2 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:window_kernel -s 1 -c 1 \
      -o $OUT/${TAG}_window_${c} -f python bench.py --config $c --algo prefix --steps 1 --warmup 1 --no-cpu-baseline > $OUT/${TAG}_ncu_${c}.log 2>&1
done
echo done
