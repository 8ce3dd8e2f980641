#!/bin/bash
# Local-linear path on the GPU box: bash tools/gpu_ll.sh TAG
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_ll.py -x -q > $OUT/${TAG}_pytest_ll.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_ll.log
for c in C2 C3 C5 C4; do
  timeout 300 python bench.py --ll --config $c --steps 5 --warmup 3 > $OUT/${TAG}_bench_ll_$c.json 2> $OUT/${TAG}_bench_ll_$c.err
done
timeout 300 python bench.py --ll --config C2 --kernel uniform --steps 5 --warmup 3 > $OUT/${TAG}_bench_ll_C2_uniform.json 2>&1
timeout 300 python bench.py --ll --config C2 --kernel triangular --steps 5 --warmup 3 > $OUT/${TAG}_bench_ll_C2_tri.json 2>&1
echo done
