#!/bin/bash
# r02bh: win_kernel preferred shared-memory carve-out (KRCV_WIN2_CARVE = 0 max L1 / 100 max smem / unset) at C2-C5
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02bh
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
for C in C2 C3 C4 C5; do
for V in unset 0 100; do
  if [ $V = unset ]; then E=""; else E="KRCV_WIN2_CARVE=$V"; fi
  env $E timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/${T}_c${V}_bench_$C.json 2> /dev/null
done
done
echo done
