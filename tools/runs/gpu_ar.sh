#!/bin/bash
# validation after the reduce/finalize shuffle trees, one-copy D2H, seg variant + nbc sweep
TAG=${1:-r01ar}; OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/${TAG}_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_gpu.log
timeout 600 python bench.py > $OUT/${TAG}_bench_C2.json 2> $OUT/${TAG}_bench_C2.err
for c in C3 C5 C4; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_$c.json 2> $OUT/${TAG}_bench_$c.err
done
for nbc in 10 16 40; do
  KRCV_WIN_NBC=$nbc timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_C2_nbc$nbc.json 2>/dev/null
done
echo done
