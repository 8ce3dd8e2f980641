#!/bin/bash
# r02u: ncu --set full of win_kernel at C2-C5 (current build) for roofline.traffic / roofline.ncu; launch list C2
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02u_build.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 3 -c 1 \
    -o $OUT/r02u_win_C2 python bench.py --config C2 --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/r02u_ncu_C2.log 2>&1
for C in C3 C4 C5; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 1 -c 1 \
    -o $OUT/r02u_win_$C python bench.py --config $C --steps 1 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/r02u_ncu_$C.log 2>&1
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02u_launches_C2.csv \
    python bench.py --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/r02u_launch_bench.log 2>&1
echo done
