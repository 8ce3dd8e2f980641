#!/bin/bash
# r02t: fused O(n) build (prefix + bucket table in one launch with a grid barrier) for <= #SMs tiles
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02t_build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window_variants.py tests/test_gpu_baseline_curves.py tests/test_gpu_property.py tests/test_gpu_host_path.py tests/test_gpu_ci.py -m gpu -x -q -p no:cacheprovider > $OUT/r02t_pytest.log 2>&1; echo "exit $?" >> $OUT/r02t_pytest.log
for C in C1 C2; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/r02t_bench_$C.json 2> $OUT/r02t_bench_$C.err
  KRCV_PFX_UNFUSED=1 timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/r02t_unfused_bench_$C.json 2> $OUT/r02t_unfused_bench_$C.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02t_launches_C2.csv \
    python bench.py --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/r02t_launch_bench.log 2>&1
timeout 900 python -m pytest tests/test_gpu_sanitizer.py -m gpu -x -q -p no:cacheprovider > $OUT/r02t_sanitizer.log 2>&1; echo "exit $?" >> $OUT/r02t_sanitizer.log
echo done
