#!/bin/bash
# r02ag: two-phase scan with ITEMS=4 staged through shared memory, terms recomputed for the stores (124 -> 62 registers)
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02ag_build.log 2>&1
KRCV_PFX_ITEMS=4 timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_ll.py tests/test_gpu_property.py -m gpu -x -q -p no:cacheprovider > $OUT/r02ag_pytest_i4.log 2>&1; echo "exit $?" >> $OUT/r02ag_pytest_i4.log
timeout 900 python -m pytest tests/test_gpu_baseline_curves.py tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider > $OUT/r02ag_pytest.log 2>&1; echo "exit $?" >> $OUT/r02ag_pytest.log
for C in C4 C5; do
  for I in default 4; do
    if [ $I = default ]; then E=""; else E="KRCV_PFX_ITEMS=$I"; fi
    env $E timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/r02ag_${I}_bench_$C.json 2> /dev/null
  done
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02ag_launches_C4.csv python bench.py --config C4 --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > /dev/null 2>&1
KRCV_PFX_ITEMS=4 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02ag_launches_C5_i4.csv python bench.py --config C5 --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > /dev/null 2>&1
echo done
