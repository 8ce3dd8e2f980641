#!/bin/bash
# r02aa: three-phase prefix build (tile totals, one-CTA offset scan, 256-record tile scan) for n above the fused size; A/B vs the 1024-record two-launch build
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02aa_build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_ll.py tests/test_gpu_property.py tests/test_gpu_ci.py -m gpu -x -q -p no:cacheprovider > $OUT/r02aa_pytest.log 2>&1; echo "exit $?" >> $OUT/r02aa_pytest.log
KRCV_PFX_ITEMS=3 timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ll.py -m gpu -x -q -p no:cacheprovider > $OUT/r02aa_pytest_3all.log 2>&1; echo "exit $?" >> $OUT/r02aa_pytest_3all.log
for C in C2 C3 C4 C5; do
  for S in default 4 1; do
    if [ $S = default ]; then E=""; else E="KRCV_PFX_ITEMS=$S"; fi
    env $E timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02aa_${S}_bench_$C.json 2> /dev/null
  done
done
echo done
