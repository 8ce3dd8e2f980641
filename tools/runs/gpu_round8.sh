#!/bin/bash
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests/test_gpu_property.py -x -q > $OUT/${TAG}_pytest_property.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_property.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/${TAG}_smoke.log 2>&1; echo "exit $?" >> $OUT/${TAG}_smoke.log
timeout 600 python bench.py > $OUT/${TAG}_bench_C2.json 2> $OUT/${TAG}_bench_C2.err
for ch in 3 1; do
  KRCV_CHUNK=$ch timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_C2_chunk$ch.json 2> /dev/null
done
echo done
