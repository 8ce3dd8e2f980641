#!/bin/bash
# r02g: win_kernel without shared memory (warp butterfly per (tile, b), lane-held sums, h by shuffle), blocked records
set -u
OUT=gpurun_out; mkdir -p $OUT
CS=paper_conf_ipps_rohlfsz17_b200/csrc
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02g_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window_variants.py tests/test_gpu_baseline_curves.py -m gpu -x -q > $OUT/r02g_pytest.log 2>&1; echo "exit $?" >> $OUT/r02g_pytest.log
for C in C2 C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --steps 10 --warmup 3 > $OUT/r02g_bench_$C.json 2> $OUT/r02g_bench_$C.err
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 3 -c 1 \
    -o $OUT/r02g_win_C2 python bench.py --config C2 --steps 2 --warmup 1 --no-alt --no-cpu-baseline > $OUT/r02g_ncu_C2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 1 -c 1 \
    -o $OUT/r02g_win_C4 python bench.py --config C4 --steps 1 --warmup 1 --no-alt --no-cpu-baseline > $OUT/r02g_ncu_C4.log 2>&1
echo done
