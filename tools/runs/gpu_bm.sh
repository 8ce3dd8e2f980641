#!/bin/bash
# host path: parallel input copies + zero-copy result block
TAG=${1:-r01bm}; OUT=gpurun_out; mkdir -p $OUT
timeout 600 python tools/e2e_overhead.py > $OUT/${TAG}_e2e_overhead.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/${TAG}_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_gpu.log
timeout 600 python bench.py > $OUT/${TAG}_bench_C2.json 2> $OUT/${TAG}_bench_C2.err
echo done
