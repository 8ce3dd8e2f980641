#!/bin/bash
# r02k: phased two-bandwidth win_kernel (ILP 2 on every memory round trip); MINB sweep 8/6/5/4
set -u
OUT=gpurun_out; mkdir -p $OUT
CS=paper_conf_ipps_rohlfsz17_b200/csrc
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02k_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window_variants.py -m gpu -x -q > $OUT/r02k_pytest.log 2>&1; echo "exit $?" >> $OUT/r02k_pytest.log
for MB in 8 6 5 4; do
  rm -f $CS/build/krcv_device.o; make -s -C $CS EXTRA=-DKRCV_WIN2_MINB=$MB > $OUT/r02k_build_mb$MB.log 2>&1
  for C in C2 C3 C4 C5; do
    timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --steps 10 --warmup 3 > $OUT/r02k_mb${MB}_bench_$C.json 2> $OUT/r02k_mb${MB}_bench_$C.err
  done
done
rm -f $CS/build/krcv_device.o; make -s -C $CS > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 1 -c 1 \
    -o $OUT/r02k_win_C4 python bench.py --config C4 --steps 1 --warmup 1 --no-alt --no-cpu-baseline > $OUT/r02k_ncu_C4.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 3 -c 1 \
    -o $OUT/r02k_win_C2 python bench.py --config C2 --steps 2 --warmup 1 --no-alt --no-cpu-baseline > $OUT/r02k_ncu_C2.log 2>&1
echo done
