#!/bin/bash
TAG=${1:-r01bk}; OUT=gpurun_out; mkdir -p $OUT
timeout 600 python -m pytest tests/test_c_consumer.py -q > $OUT/${TAG}_pytest_c.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_c.log
echo done
