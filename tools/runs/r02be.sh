#!/bin/bash
# r02be: win_kernel minimum chunk (bandwidths per task) at C2 / C1 / C3 after the per-task overhead cuts:
# KRCV_WIN2_MINCHUNK = 1 / 2 / 3 (default) / 4, twice each
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02be
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
for rep in 1 2; do
for C in C2 C1; do
for V in 1 2 3 4; do
  KRCV_WIN2_MINCHUNK=$V timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 30 --warmup 5 > $OUT/${T}_mc${V}_r${rep}_bench_$C.json 2> /dev/null
done
done
done
for V in 1 3; do
  KRCV_WIN2_MINCHUNK=$V timeout 300 python bench.py --config C3 --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/${T}_mc${V}_bench_C3.json 2> /dev/null
done
echo done
