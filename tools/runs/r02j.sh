#!/bin/bash
# r02j: finer win_kernel tasks (>= 8 per slot, BC >= 1), bucket fill with 8 items per thread
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02j_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window_variants.py -m gpu -x -q > $OUT/r02j_pytest.log 2>&1; echo "exit $?" >> $OUT/r02j_pytest.log
for C in C2 C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --steps 10 --warmup 3 > $OUT/r02j_bench_$C.json 2> $OUT/r02j_bench_$C.err
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02j_launches_C2.csv \
    python bench.py --steps 2 --warmup 1 --no-alt --no-cpu-baseline > $OUT/r02j_launch_bench.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02j_launches_C5.csv \
    python bench.py --config C5 --steps 2 --warmup 1 --no-alt --no-cpu-baseline > $OUT/r02j_launch_bench5.log 2>&1
echo done
