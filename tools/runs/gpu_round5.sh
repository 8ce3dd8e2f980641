#!/bin/bash
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/${TAG}_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_gpu.log
timeout 600 python bench.py > $OUT/${TAG}_bench_C2.json 2> $OUT/${TAG}_bench_C2.err
for c in C3 C5 C4; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > $OUT/${TAG}_bench_$c.json 2> $OUT/${TAG}_bench_$c.err
done
for c in C2 C3 C5; do
  timeout 300 python bench.py --ll --config $c --steps 10 --warmup 3 > $OUT/${TAG}_bench_ll_$c.json 2>&1
  timeout 300 python bench.py --kde --config $c --steps 10 --warmup 3 > $OUT/${TAG}_bench_kde_$c.json 2>&1
done
echo done
