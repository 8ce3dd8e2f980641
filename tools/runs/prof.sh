#!/bin/bash
# ncu --set full capture of the sweep kernel: bash tools/prof.sh TAG CONFIG [G]
OUT=gpurun_out; mkdir -p $OUT; TAG=$1; C=$2; G=${3:-}
export KRCV_SWEEP_G=$G
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 1 -c 1 \
    -o $OUT/${TAG}_sweep_${C} -f python bench.py --config $C --steps 1 --warmup 1 --no-cpu-baseline > $OUT/${TAG}_ncu_${C}.log 2>&1
echo "ncu exit $?" >> $OUT/${TAG}_ncu_${C}.log
