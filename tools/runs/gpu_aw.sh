#!/bin/bash
TAG=${1:-r01ay}; OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_baseline_curves.py -q -s > $OUT/${TAG}_pytest_curves.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_curves.log
timeout 900 python tools/parity_report.py $OUT/${TAG}_parity_report.md > $OUT/${TAG}_parity_report.log 2>&1
timeout 600 python bench.py > $OUT/${TAG}_bench_C2.json 2> $OUT/${TAG}_bench_C2.err
echo done
