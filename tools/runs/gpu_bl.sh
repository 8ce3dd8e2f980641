#!/bin/bash
TAG=${1:-r01bl}; OUT=gpurun_out; mkdir -p $OUT
timeout 600 python tools/e2e_overhead.py > $OUT/${TAG}_e2e_overhead.txt 2>&1
echo done
