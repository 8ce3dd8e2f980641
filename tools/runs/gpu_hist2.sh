#!/bin/bash
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_hist.py tests/test_gpu_ll.py -x -q > $OUT/${TAG}_pytest_hist_ll.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_hist_ll.log
KRCV_LL_STATS=1 timeout 300 python bench.py --ll --config C5 --steps 1 --warmup 0 > $OUT/${TAG}_ll_stats_C5.txt 2>&1
for c in C2 C3 C5 C4; do
  timeout 300 python bench.py --ll --config $c --steps 5 --warmup 3 > $OUT/${TAG}_bench_ll_$c.json 2> $OUT/${TAG}_bench_ll_$c.err
done
timeout 600 python bench.py --config C2 --algo hist --steps 5 --warmup 3 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_C2_hist.json 2> $OUT/${TAG}_bench_C2_hist.err
timeout 900 ncu --set full --clock-control none --import-source on -k regex:hist_kernel -s 1 -c 1 \
    -o $OUT/${TAG}_hist_C2 -f python bench.py --config C2 --algo hist --steps 1 --warmup 1 --no-cpu-baseline --no-alt > $OUT/${TAG}_ncu_hist.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:ll_window_kernel -s 1 -c 1 \
    -o $OUT/${TAG}_ll_C3 -f python bench.py --ll --config C3 --steps 1 --warmup 1 > $OUT/${TAG}_ncu_ll.log 2>&1
echo done
