#!/bin/bash
TAG=${1:-r01ba}; OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "kde" > $OUT/${TAG}_pytest_kde.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_kde.log
for c in C2 C3 C5; do for k in epanechnikov uniform triangular; do
  timeout 300 python bench.py --kde --config $c --kernel $k --steps 10 --warmup 3 > $OUT/${TAG}_bench_kde_${c}_$k.json 2> $OUT/${TAG}_bench_kde_${c}_$k.err
done; done
echo done
for c in C2 C3 C5; do for k in epanechnikov uniform triangular; do
  KRCV_LIB=$PWD/tools/libkrcv_base.bin timeout 300 python bench.py --kde --config $c --kernel $k --steps 10 --warmup 3 > $OUT/${TAG}_base_kde_${c}_$k.json 2> $OUT/${TAG}_base_kde_${c}_$k.err
done; done
