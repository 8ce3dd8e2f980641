#!/bin/bash
# r02ba: end-of-round validation of HEAD (schedule constants as parameters, 16-anchor rule) -- full GPU suite, smoke, default bench, reference arm, parity table, launch lists, ncu of win_kernel at C2-C5
# reference arm, parity table, C2/C4 launch lists, ncu --set full of win_kernel at C2-C5
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02ba
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/${T}_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
timeout 3000 python -m pytest tests -m gpu -x -q -p no:cacheprovider > $OUT/${T}_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/${T}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/${T}_smoke.log 2>&1; echo "exit $?" >> $OUT/${T}_smoke.log
timeout 900 python bench.py > $OUT/${T}_bench_default.json 2> $OUT/${T}_bench_default.err
timeout 600 python bench.py --impl reference > $OUT/${T}_bench_reference.json 2> $OUT/${T}_bench_reference.err
timeout 1200 python tools/parity_report.py $OUT/${T}_parity_report.md > $OUT/${T}_parity_report.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/${T}_launches_C2.csv \
    python bench.py --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/${T}_launch_bench.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/${T}_launches_C4.csv \
    python bench.py --config C4 --steps 1 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/${T}_launch_bench_C4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 3 -c 1 \
    -o $OUT/${T}_win_C2 python bench.py --config C2 --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/${T}_ncu_C2.log 2>&1
for C in C3 C4 C5; do
timeout 900 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 1 -c 1 \
    -o $OUT/${T}_win_$C python bench.py --config $C --steps 1 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/${T}_ncu_$C.log 2>&1
done
echo done
