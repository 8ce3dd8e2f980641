#!/bin/bash
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/${TAG}_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_gpu.log
timeout 600 python bench.py > $OUT/${TAG}_bench_C2.json 2> $OUT/${TAG}_bench_C2.err
KRCV_PFX_TWO=1 timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_C2_pfx2.json 2> /dev/null
for c in C3 C5 C4; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > $OUT/${TAG}_bench_$c.json 2> $OUT/${TAG}_bench_$c.err
  KRCV_PFX_TWO=1 timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_pfx2.json 2> /dev/null
done
timeout 300 python bench.py --ll --config C2 --steps 10 --warmup 3 > $OUT/${TAG}_bench_ll_C2.json 2>&1
timeout 300 python bench.py --kde --config C2 --steps 10 --warmup 3 > $OUT/${TAG}_bench_kde_C2.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/${TAG}_launches_C2.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-alt > $OUT/${TAG}_ncu_launch_bench.log 2>&1
echo done
