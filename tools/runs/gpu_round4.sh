#!/bin/bash
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "graph" > $OUT/${TAG}_pytest_gpu_sub.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_gpu_sub.log
timeout 600 python bench.py > $OUT/${TAG}_bench_C2.json 2> $OUT/${TAG}_bench_C2.err
for c in C3 C5 C4; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > $OUT/${TAG}_bench_$c.json 2> $OUT/${TAG}_bench_$c.err
done
for c in C4 C5; do for NBC in 1 2 4 8; do
  KRCV_WIN_NBC=$NBC timeout 300 python bench.py --config $c --steps 5 --warmup 2 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_nbc$NBC.json 2>/dev/null
done; done
for c in C2 C3; do for K in 1 3; do
  KRCV_WIN_K=$K timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_K$K.json 2>/dev/null
done; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/${TAG}_launches_C2.csv \
    python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-alt > $OUT/${TAG}_ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:window_kernel -s 2 -c 1 \
    -o $OUT/${TAG}_window_C2 -f python bench.py --steps 1 --warmup 2 --no-cpu-baseline --no-alt > $OUT/${TAG}_ncu_full.log 2>&1
echo done
