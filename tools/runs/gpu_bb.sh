#!/bin/bash
TAG=${1:-r01bb}; OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "max_grid or kde" > $OUT/${TAG}_pytest.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest.log
for c in C2 C3 C5; do
  timeout 300 python bench.py --kde --config $c --steps 10 --warmup 3 > $OUT/${TAG}_bench_kde_$c.json 2> $OUT/${TAG}_bench_kde_$c.err
  timeout 300 python bench.py --ll --config $c --steps 10 --warmup 3 > $OUT/${TAG}_bench_ll_$c.json 2> $OUT/${TAG}_bench_ll_$c.err
done
timeout 300 python bench.py --kernel gaussian --steps 3 --warmup 3 --no-cpu-baseline > $OUT/${TAG}_bench_C2_gaussian.json 2> $OUT/${TAG}_bench_C2_gaussian.err
echo done
