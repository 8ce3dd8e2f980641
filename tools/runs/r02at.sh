#!/bin/bash
# r02at: merge-path chunk-pair rank counts (rank_merge_kernel) vs r02's ordered-pair binary searches: sort-variant
# tests (every a2 implementation bit-identical), parity, C1-C3 bench A/B, C2 launch list
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02at
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_sort_variants.py tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider > $OUT/${T}_pytest.log 2>&1; echo "exit $?" >> $OUT/${T}_pytest.log
for C in C1 C2 C3; do
  for V in merge bsearch; do
    if [ $V = bsearch ]; then E="KRCV_RANK_BSEARCH=1"; else E=""; fi
    env $E timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 30 --warmup 5 > $OUT/${T}_${V}_bench_$C.json 2> /dev/null
  done
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/${T}_launches_C2.csv \
    python bench.py --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/${T}_launch_bench.log 2>&1
echo done
