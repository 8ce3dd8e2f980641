#!/bin/bash
# r02ac: three-phase prefix build v2 (round-based one-CTA offset scan; ITEMS 1 or 4) vs two-phase; parity with 3P forced at ITEMS 1 and 4
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02ac_build.log 2>&1
KRCV_PFX_3P=1 KRCV_PFX_ITEMS=1 timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_ll.py -m gpu -x -q -p no:cacheprovider > $OUT/r02ac_pytest_3p1.log 2>&1; echo "exit $?" >> $OUT/r02ac_pytest_3p1.log
KRCV_PFX_3P=1 KRCV_PFX_ITEMS=4 timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_ll.py -m gpu -x -q -p no:cacheprovider > $OUT/r02ac_pytest_3p4.log 2>&1; echo "exit $?" >> $OUT/r02ac_pytest_3p4.log
for C in C3 C4 C5; do
  for I in 1 4; do
    for P in 0 1; do
      KRCV_PFX_ITEMS=$I KRCV_PFX_3P=$P timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02ac_i${I}p${P}_bench_$C.json 2> /dev/null
    done
  done
done
KRCV_PFX_ITEMS=4 KRCV_PFX_3P=1 timeout 600 ncu --set full --import-source on --clock-control none -k regex:pfx_ -c 3 -o $OUT/r02ac_pfx3_C4 python bench.py --config C4 --no-alt --no-cpu-baseline --no-extra --steps 1 --warmup 0 > /dev/null 2>&1
echo done
