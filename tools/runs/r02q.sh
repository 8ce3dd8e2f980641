#!/bin/bash
# r02q: a5 (column sums + finalize) fused into win_kernel via per-chunk completion counters
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02q_build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window_variants.py tests/test_gpu_distributed.py tests/test_gpu_faults.py tests/test_gpu_baseline_curves.py tests/test_gpu_host_path.py -m gpu -x -q -p no:cacheprovider > $OUT/r02q_pytest.log 2>&1; echo "exit $?" >> $OUT/r02q_pytest.log
for C in C2 C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02q_bench_$C.json 2> $OUT/r02q_bench_$C.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02q_launches_C2.csv \
    python bench.py --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/r02q_launch_bench.log 2>&1
echo done
