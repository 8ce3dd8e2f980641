#!/bin/bash
# r02z: 32-bit quantised-key sort (4 radix passes + exact run fix-up) for n > 131,072; A/B vs CUB 64-bit and the rank sort
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02z_build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_window_variants.py tests/test_gpu_sweep_gxg.py -m gpu -x -q -p no:cacheprovider > $OUT/r02z_pytest.log 2>&1; echo "exit $?" >> $OUT/r02z_pytest.log
KRCV_SORT=q32 timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window_variants.py -m gpu -x -q -p no:cacheprovider > $OUT/r02z_pytest_q32all.log 2>&1; echo "exit $?" >> $OUT/r02z_pytest_q32all.log
for C in C3 C4 C5; do
  for S in default q32 cub64 rank; do
    if [ $S = rank ] && [ $C != C3 ]; then continue; fi
    KRCV_SORT=$S timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02z_${S}_bench_$C.json 2> /dev/null
  done
done
KRCV_SORT=q32 timeout 300 python bench.py --config C2 --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02z_q32_bench_C2.json 2> /dev/null
echo done
