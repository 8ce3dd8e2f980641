#!/bin/bash
TAG=${1:-r01bi}; OUT=gpurun_out; mkdir -p $OUT
timeout 900 python tools/shard_balance.py C2 C3 C5 C4 > $OUT/${TAG}_shard_balance.txt 2>&1
echo done
