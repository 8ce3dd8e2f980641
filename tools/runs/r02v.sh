#!/bin/bash
# r02v: task granularity (KRCV_WIN2_TPW) at C2/C3/C5; two running sums per lane (64-bandwidth chunks) at C3-C5
set -u
OUT=gpurun_out; mkdir -p $OUT
CS=paper_conf_ipps_rohlfsz17_b200/csrc
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02v_build.log 2>&1
for T in 2 4 8 16; do
  for C in C2 C3 C5; do
    KRCV_WIN2_TPW=$T timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02v_tpw${T}_bench_$C.json 2> /dev/null
  done
done
rm -f $CS/build/krcv_device.o; make -s -C $CS EXTRA=-DKRCV_WIN2_ACC=2 > $OUT/r02v_build_acc2.log 2>&1
timeout 600 python -m pytest tests/test_gpu_window_variants.py -m gpu -x -q -k oracle -p no:cacheprovider > $OUT/r02v_pytest_acc2.log 2>&1; echo "exit $?" >> $OUT/r02v_pytest_acc2.log
for C in C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02v_acc2_bench_$C.json 2> /dev/null
done
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:win_kernel -s 1 -c 1 --csv --log-file $OUT/r02v_acc2_dram_C4.csv \
    python bench.py --config C4 --steps 1 --warmup 1 --no-alt --no-cpu-baseline --no-extra > /dev/null 2>&1
rm -f $CS/build/krcv_device.o; make -s -C $CS > /dev/null 2>&1
echo done
