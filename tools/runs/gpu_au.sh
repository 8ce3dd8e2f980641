#!/bin/bash
TAG=${1:-r01au}; OUT=gpurun_out; mkdir -p $OUT
timeout 2400 python -m pytest tests/test_gpu_sanitizer.py -q -x --durations=0 > $OUT/${TAG}_pytest_sanitizer.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_sanitizer.log
echo done
