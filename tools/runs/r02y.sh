#!/bin/bash
# r02y: bucket-table cap (kBktFmax 32 / 16 / 8) at C5 (heavy tail, where F hits the cap) and C2
set -u
OUT=gpurun_out; mkdir -p $OUT
CS=paper_conf_ipps_rohlfsz17_b200/csrc
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02y_build.log 2>&1
for F in 32 16 8 4; do
  rm -f $CS/build/krcv_device.o; make -s -C $CS EXTRA=-DKRCV_BKT_FMAX=$F > $OUT/r02y_build_f$F.log 2>&1
  for C in C5 C2; do
    timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02y_f${F}_bench_$C.json 2> /dev/null
  done
done
rm -f $CS/build/krcv_device.o; make -s -C $CS > /dev/null 2>&1
echo done
