#!/bin/bash
# cost-balanced row cuts: row-range ABI tests, multi-rank balanced path, balance emulation on one GPU
TAG=${1:-r01bh}; OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_distributed.py -q -x -k "row_ranges or sharded or shard" > $OUT/${TAG}_pytest.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest.log
timeout 900 python tools/shard_balance.py C2 C3 C5 C4 > $OUT/${TAG}_shard_balance.txt 2>&1
KRCV_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 \
  bench.py --gpus 2 --steps 5 --warmup 3 > $OUT/${TAG}_bench_2ranks_gloo.json 2> $OUT/${TAG}_bench_2ranks_gloo.err
echo done
