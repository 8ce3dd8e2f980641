#!/bin/bash
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02r_build.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 3 -c 1 \
    -o $OUT/r02r_win_C2 python bench.py --config C2 --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/r02r_ncu_C2.log 2>&1
echo done
