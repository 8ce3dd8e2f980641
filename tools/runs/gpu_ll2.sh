#!/bin/bash
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_ll.py tests/test_gpu_property.py -x -q -k "ll or local" > $OUT/${TAG}_pytest_ll.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_ll.log
for c in C2 C5; do KRCV_LL_STATS=1 timeout 300 python bench.py --ll --config $c --steps 1 --warmup 0 > $OUT/${TAG}_ll_stats_$c.txt 2>&1; done
for c in C2 C3 C5 C4; do
  timeout 300 python bench.py --ll --config $c --steps 5 --warmup 3 > $OUT/${TAG}_bench_ll_$c.json 2> $OUT/${TAG}_bench_ll_$c.err
done
timeout 300 python bench.py --ll --config C2 --kernel uniform --steps 5 --warmup 3 > $OUT/${TAG}_bench_ll_C2_uniform.json 2>&1
echo done
