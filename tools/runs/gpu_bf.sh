#!/bin/bash
# 128- vs 256-record prefix tiles (one-item build, 1,024 < n <= 2^18)
TAG=${1:-r01bf}; OUT=gpurun_out; mkdir -p $OUT
for T in 128 256; do for c in C2 C3 C5; do
  KRCV_PFX_THREADS=$T timeout 300 python bench.py --config $c --steps 20 --warmup 5 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_T$T.json 2>/dev/null
done; done
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ll.py tests/test_gpu_baseline_curves.py -x -q > $OUT/${TAG}_pytest.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest.log
echo done
