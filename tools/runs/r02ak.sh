#!/bin/bash
# r02ak: smaller win_kernel chunks when the slots are under-filled (C1); fused O(n) build at n <= 1024 (KRCV_PFX_ITEMS=1) vs the one-CTA build; full GPU suite
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02ak_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -x -q -p no:cacheprovider > $OUT/r02ak_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/r02ak_pytest_gpu.log
for V in default i1; do
  if [ $V = default ]; then E=""; else E="KRCV_PFX_ITEMS=1"; fi
  env $E timeout 300 python bench.py --config C1 --no-alt --no-cpu-baseline --no-extra --steps 30 --warmup 5 > $OUT/r02ak_${V}_bench_C1.json 2> /dev/null
done
timeout 300 python bench.py --config C2 --no-alt --no-cpu-baseline --no-extra --steps 30 --warmup 5 > $OUT/r02ak_default_bench_C2.json 2> /dev/null
echo done
