#!/bin/bash
# r02c: ncu --set full of win_kernel at C2 and C4 (source-level), launch list at C2
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02c_build.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 3 -c 1 \
    -o $OUT/r02c_win_C2 python bench.py --config C2 --steps 2 --warmup 1 --no-alt --no-cpu-baseline > $OUT/r02c_ncu_C2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 1 -c 1 \
    -o $OUT/r02c_win_C4 python bench.py --config C4 --steps 1 --warmup 1 --no-alt --no-cpu-baseline > $OUT/r02c_ncu_C4.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02c_launches_C2.csv \
    python bench.py --steps 2 --warmup 1 --no-alt --no-cpu-baseline > $OUT/r02c_launch_bench.log 2>&1
echo done
