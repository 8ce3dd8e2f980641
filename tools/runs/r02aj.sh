#!/bin/bash
# (the balance rule it measured was not kept; the C1 rule for under-filled slots is)
# r02aj: win_kernel chunk size chosen for slot balance (min ceil(tasks/S)(BC + c0)) vs round 2's 16-tasks-per-slot rule
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02aj_build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_window_variants.py tests/test_gpu_ci.py -m gpu -x -q -p no:cacheprovider > $OUT/r02aj_pytest.log 2>&1; echo "exit $?" >> $OUT/r02aj_pytest.log
for C in C2 C3 C5 C4 C1; do
  for V in old c1 c05 c2 c4; do
    case $V in
      old) E="KRCV_WIN2_TPW=16";; c1) E="KRCV_WIN2_C0=1";; c05) E="KRCV_WIN2_C0=0.5";; c2) E="KRCV_WIN2_C0=2";; c4) E="KRCV_WIN2_C0=4";;
    esac
    env $E timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/r02aj_${V}_bench_$C.json 2> /dev/null
  done
done
echo done
