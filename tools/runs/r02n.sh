#!/bin/bash
# r02n: launch lists at C3, C4, C5 (default path) and the sort-path A/B at C3 (chunk-rank vs CUB)
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02n_build.log 2>&1
for C in C3 C4 C5; do
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02n_launches_$C.csv \
    python bench.py --config $C --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/r02n_launch_$C.log 2>&1
done
for C in C2 C3; do
  KRCV_CUB_SORT=1 timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02n_cub_bench_$C.json 2> $OUT/r02n_cub_bench_$C.err
done
echo done
