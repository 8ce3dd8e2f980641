#!/bin/bash
# r02s: prefix-build tile size at C4/C5 (ITEMS 1 vs 4), bucket factor cap at C5, and the N>1 bench path
# (torchrun, 2 ranks on one GPU over gloo: eager fallback, shard + all-reduce + finalize)
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02s_build.log 2>&1
for C in C4 C5; do
  KRCV_PFX_ITEMS=1 timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02s_items1_bench_$C.json 2> $OUT/r02s_items1_bench_$C.err
  KRCV_PFX_ITEMS=4 timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02s_items4_bench_$C.json 2> $OUT/r02s_items4_bench_$C.err
done
KRCV_BENCH_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29555 \
  bench.py --gpus 2 --steps 5 --warmup 3 > $OUT/r02s_bench_2ranks_gloo.json 2> $OUT/r02s_bench_2ranks_gloo.err
echo "exit $?" >> $OUT/r02s_bench_2ranks_gloo.err
echo done
