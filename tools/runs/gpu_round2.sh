#!/bin/bash
# full GPU tests + benches on C2-C5 + LL/KDE: bash tools/gpu_round2.sh TAG
TAG=${1:-r01}; OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/${TAG}_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/${TAG}_smoke.log 2>&1; echo "exit $?" >> $OUT/${TAG}_smoke.log
timeout 600 python bench.py > $OUT/${TAG}_bench_C2.json 2> $OUT/${TAG}_bench_C2.err
for c in C3 C5 C4; do
  timeout 600 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline > $OUT/${TAG}_bench_$c.json 2> $OUT/${TAG}_bench_$c.err
done
for c in C4 C5; do for NBC in 1 2 4 8; do
  KRCV_WIN_NBC=$NBC timeout 300 python bench.py --config $c --steps 5 --warmup 2 --no-cpu-baseline --no-alt > $OUT/${TAG}_bench_${c}_nbc$NBC.json 2>/dev/null
done; done
timeout 300 python bench.py --ll --config C2 --steps 10 --warmup 3 > $OUT/${TAG}_bench_ll_C2.json 2>&1
timeout 300 python bench.py --kde --config C2 --steps 10 --warmup 3 > $OUT/${TAG}_bench_kde_C2.json 2>&1
echo done
