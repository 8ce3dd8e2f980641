#!/bin/bash
# r02o: win_kernel build-time A/B: records AoS vs blocked, bucket factor, rows per lane, division
set -u
OUT=gpurun_out; mkdir -p $OUT
CS=paper_conf_ipps_rohlfsz17_b200/csrc
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02o_build.log 2>&1
declare -A V
V[v0]=""
V[v1]="-DKRCV_REC_AOS=1"
V[v2]="-DKRCV_BKT_FX=2.0"
V[v3]="-DKRCV_WIN2_ROWS=1"
V[v4]="-DKRCV_FASTDIV=0"
V[v5]="-DKRCV_REC_AOS=1 -DKRCV_BKT_FX=2.0 -DKRCV_WIN2_ROWS=1"
V[v6]="-DKRCV_REC_AOS=1 -DKRCV_BKT_FX=2.0"
for k in v0 v1 v2 v3 v4 v5 v6; do
  rm -f $CS/build/krcv_device.o; make -s -C $CS EXTRA="${V[$k]}" > $OUT/r02o_build_$k.log 2>&1
  timeout 600 python -m pytest tests/test_gpu_window_variants.py -m gpu -x -q -k oracle -p no:cacheprovider > $OUT/r02o_pytest_$k.log 2>&1; echo "exit $?" >> $OUT/r02o_pytest_$k.log
  for C in C2 C3 C4 C5; do
    timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02o_${k}_bench_$C.json 2> $OUT/r02o_${k}_bench_$C.err
  done
done
rm -f $CS/build/krcv_device.o; make -s -C $CS > /dev/null 2>&1
echo done
