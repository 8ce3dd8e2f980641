#!/bin/bash
# r02al: fused O(n) build also at n <= 1,024 (regression moment sets); full GPU suite, smoke, C1/C2 bench
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02al_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider > $OUT/r02al_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/r02al_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/r02al_smoke.log 2>&1; echo "exit $?" >> $OUT/r02al_smoke.log
for C in C1 C2; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 30 --warmup 5 > $OUT/r02al_bench_$C.json 2> /dev/null
done
echo done
