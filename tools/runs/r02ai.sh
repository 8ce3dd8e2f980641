#!/bin/bash
# (the cluster rank sort this script measured was removed after the run)
# r02ai: cluster rank sort (chunk sorts in 8-CTA clusters, group ranks over distributed shared memory, global ranks + scatter) vs the chunk-pair rank sort
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02ai_build.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_sanitizer.py tests/test_gpu_host_path.py tests/test_gpu_faults.py -m gpu -x -q -p no:cacheprovider > $OUT/r02ai_pytest.log 2>&1; echo "exit $?" >> $OUT/r02ai_pytest.log
for C in C1 C2 C3; do
  for S in cluster rank; do
    KRCV_SORT=$S timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/r02ai_${S}_bench_$C.json 2> /dev/null
  done
done
for CH in 3 0; do
  KRCV_SORT=cluster KRCV_CHUNK=$CH timeout 300 python bench.py --config C2 --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/r02ai_cluster_ch${CH}_bench_C2.json 2> /dev/null
  KRCV_SORT=cluster KRCV_CHUNK=$CH timeout 300 python bench.py --config C3 --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/r02ai_cluster_ch${CH}_bench_C3.json 2> /dev/null
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02ai_launches_C2.csv python bench.py --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02ai_launches_C3.csv python bench.py --config C3 --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > /dev/null 2>&1
echo done
