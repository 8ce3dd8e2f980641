#!/bin/bash
# one-CTA prefix build for n <= 2^15 (KRCV_PFX_ITEMS=0, default there) vs the two-phase build (=1)
TAG=${1:-r01be}; OUT=gpurun_out; mkdir -p $OUT
for P in 0 1; do for c in C2 C1; do
  KRCV_PFX_ITEMS=$P timeout 300 python bench.py --config $c --steps 20 --warmup 5 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_P$P.json 2>/dev/null
done; done
for P in 0 1; do
  KRCV_PFX_ITEMS=$P timeout 300 python bench.py --ll --config C2 --steps 10 --warmup 3 > $OUT/${TAG}_bench_ll_C2_P$P.json 2>/dev/null
  KRCV_PFX_ITEMS=$P timeout 300 python bench.py --kde --config C2 --steps 10 --warmup 3 > $OUT/${TAG}_bench_kde_C2_P$P.json 2>/dev/null
done
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/${TAG}_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_gpu.log
echo done
