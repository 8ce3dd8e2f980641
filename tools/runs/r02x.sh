#!/bin/bash
# r02x: task shape (16 tasks per slot, chunks >= 3 bandwidths): parity + bench C1-C5
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02x_build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window_variants.py tests/test_gpu_baseline_curves.py -m gpu -x -q -p no:cacheprovider > $OUT/r02x_pytest.log 2>&1; echo "exit $?" >> $OUT/r02x_pytest.log
for C in C1 C2 C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02x_bench_$C.json 2> /dev/null
done
echo done
