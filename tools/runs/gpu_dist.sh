#!/bin/bash
# multi-rank device path on one GPU (gloo): bash tools/gpu_dist.sh TAG
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_distributed.py -x -q > $OUT/${TAG}_pytest_dist.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_dist.log
KRCV_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
    bench.py --gpus 2 --steps 3 --warmup 3 > $OUT/${TAG}_bench_gloo2.json 2> $OUT/${TAG}_bench_gloo2.err; echo "exit $?" >> $OUT/${TAG}_bench_gloo2.err
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29534 \
    bench.py --gpus 2 --impl reference --steps 1 --warmup 0 > $OUT/${TAG}_bench_ref2.json 2> $OUT/${TAG}_bench_ref2.err; echo "exit $?" >> $OUT/${TAG}_bench_ref2.err
echo done
