#!/bin/bash
# r02b: first run of win_kernel (bucket-table lookups): parity subset + bench C2-C5
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02b_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window_variants.py tests/test_gpu_baseline_curves.py -m gpu -x -q > $OUT/r02b_pytest.log 2>&1; echo "exit $?" >> $OUT/r02b_pytest.log
for C in C2 C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --steps 10 --warmup 3 > $OUT/r02b_bench_$C.json 2> $OUT/r02b_bench_$C.err
done
echo done
