#!/bin/bash
# multi-rank bench path on one GPU (gloo backend, 2 ranks) + reference arm under torchrun
TAG=${1:-r01bg}; OUT=gpurun_out; mkdir -p $OUT
KRCV_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 \
  bench.py --gpus 2 --steps 5 --warmup 3 > $OUT/${TAG}_bench_2ranks_gloo.json 2> $OUT/${TAG}_bench_2ranks_gloo.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29512 \
  bench.py --impl reference --gpus 2 --steps 3 --warmup 3 > $OUT/${TAG}_bench_reference_2ranks.json 2> $OUT/${TAG}_bench_reference_2ranks.err
echo done
