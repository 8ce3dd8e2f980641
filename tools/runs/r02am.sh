#!/bin/bash
# r02am: win_kernel next-bandwidth hint prefetch (KRCV_WIN2_PF) and grouped 4-bandwidth warp reduction
# (KRCV_WIN2_TR) -- build-time A/B against the r02al kernel (PF=0, TR=1), window-variant parity for each
set -u
OUT=gpurun_out; mkdir -p $OUT
CS=paper_conf_ipps_rohlfsz17_b200/csrc
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02am_build.log 2>&1
declare -A V
V[new]=""
V[old]="-DKRCV_WIN2_PF=0 -DKRCV_WIN2_TR=1"
V[pf]="-DKRCV_WIN2_TR=1"
V[tr]="-DKRCV_WIN2_PF=0"
V[mb7]="-DKRCV_WIN2_MINB=7"
V[r1]="-DKRCV_WIN2_ROWS=1"
for k in new old pf tr mb7 r1; do
  rm -f $CS/build/krcv_device.o; make -s -C $CS EXTRA="${V[$k]}" > $OUT/r02am_build_$k.log 2>&1
  timeout 600 python -m pytest tests/test_gpu_window_variants.py -m gpu -x -q -k oracle -p no:cacheprovider > $OUT/r02am_pytest_$k.log 2>&1; echo "exit $?" >> $OUT/r02am_pytest_$k.log
  for C in C2 C3 C4 C5; do
    timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02am_${k}_bench_$C.json 2> $OUT/r02am_${k}_bench_$C.err
  done
done
rm -f $CS/build/krcv_device.o; make -s -C $CS > /dev/null 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_ci.py -m gpu -x -q -p no:cacheprovider > $OUT/r02am_pytest_parity.log 2>&1; echo "exit $?" >> $OUT/r02am_pytest_parity.log
echo done
