#!/bin/bash
# r02ap: ncu --set full of win_kernel at C2 with the anchored records (J = 1, 8) and without (J = 0): why J = 1 is slower
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02ap
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
for J in 0 1 8; do
KRCV_ANCHORS=$J timeout 600 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 3 -c 1 \
    -o $OUT/${T}_win_C2_j$J python bench.py --config C2 --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/${T}_ncu_C2_j$J.log 2>&1
done
for J in 0 8; do
KRCV_ANCHORS=$J timeout 300 python bench.py --config C2 --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/${T}_j${J}_bench_C2.json 2> /dev/null
done
echo done
