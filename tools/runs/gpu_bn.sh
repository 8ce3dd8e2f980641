#!/bin/bash
# programmatic dependent launch on/off
TAG=${1:-r01bn}; OUT=gpurun_out; mkdir -p $OUT
for P in 1 0; do for c in C2 C1 C3 C5; do
  KRCV_PDL=$P timeout 300 python bench.py --config $c --steps 20 --warmup 5 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_pdl$P.json 2>/dev/null
done; done
timeout 600 python tools/e2e_overhead.py > $OUT/${TAG}_e2e_overhead.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/${TAG}_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_gpu.log
echo done
