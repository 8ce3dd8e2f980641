#!/bin/bash
# r02bd: functional check of the N = 2 bench path (two ranks on the one GPU over gloo -- not a timing) at C2 and C3
# (C3: shard-local anchored copies, cost-balanced cuts), end-of-round build
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02bd
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
for C in C2 C3; do
KRCV_BENCH_BACKEND=gloo timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29533 bench.py --gpus 2 --config $C --steps 5 --warmup 3 --no-alt --no-cpu-baseline > $OUT/${T}_bench_2ranks_$C.json 2> $OUT/${T}_bench_2ranks_$C.err
echo "exit $?" >> $OUT/${T}_bench_2ranks_$C.err
done
echo done
