#!/bin/bash
# r02d: win_kernel with blocked double2 records, fast division, batched smem reduction:
# parity subset, bench C2-C5, register-cap sweep (KRCV_WIN2_MINB 4/6/8), ncu C2
set -u
OUT=gpurun_out; mkdir -p $OUT
CS=paper_conf_ipps_rohlfsz17_b200/csrc
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02d_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window_variants.py tests/test_gpu_baseline_curves.py -m gpu -x -q > $OUT/r02d_pytest.log 2>&1; echo "exit $?" >> $OUT/r02d_pytest.log
for C in C2 C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --steps 10 --warmup 3 > $OUT/r02d_bench_$C.json 2> $OUT/r02d_bench_$C.err
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:win_kernel -s 3 -c 1 \
    -o $OUT/r02d_win_C2 python bench.py --config C2 --steps 2 --warmup 1 --no-alt --no-cpu-baseline > $OUT/r02d_ncu_C2.log 2>&1
for MB in 4 8; do
  rm -f $CS/build/krcv_device.o; make -s -C $CS EXTRA=-DKRCV_WIN2_MINB=$MB > $OUT/r02d_build_mb$MB.log 2>&1
  for C in C2 C4 C5; do
    timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --steps 10 --warmup 3 > $OUT/r02d_mb${MB}_bench_$C.json 2> $OUT/r02d_mb${MB}_bench_$C.err
  done
done
rm -f $CS/build/krcv_device.o; make -s -C $CS > /dev/null 2>&1
echo done
