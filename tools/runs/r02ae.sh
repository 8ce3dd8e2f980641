#!/bin/bash
# r02ae: bucket-table fill with coalesced stores (tile staged in shared memory); pack_range with one atomic per CTA
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02ae_build.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_window_variants.py tests/test_gpu_sanitizer.py -m gpu -x -q -p no:cacheprovider > $OUT/r02ae_pytest.log 2>&1; echo "exit $?" >> $OUT/r02ae_pytest.log
KRCV_SORT=q32 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider > $OUT/r02ae_pytest_q32.log 2>&1; echo "exit $?" >> $OUT/r02ae_pytest_q32.log
for C in C2 C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/r02ae_bench_$C.json 2> /dev/null
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02ae_launches_C5.csv python bench.py --config C5 --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02ae_launches_C4.csv python bench.py --config C4 --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > /dev/null 2>&1
echo done
