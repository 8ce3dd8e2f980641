#!/bin/bash
# r02bf: anchor_kernel with one thread per index for all its copies (P[k] read once): anchor + window-variant +
# parity tests; C3-C5 benches; C4 launch list
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02bf
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_anchors.py tests/test_gpu_window_variants.py tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider > $OUT/${T}_pytest.log 2>&1; echo "exit $?" >> $OUT/${T}_pytest.log
for C in C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/${T}_bench_$C.json 2> /dev/null
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/${T}_launches_C4.csv \
    python bench.py --config C4 --steps 1 --warmup 1 --no-alt --no-cpu-baseline --no-extra > $OUT/${T}_launch_bench_C4.log 2>&1
echo done
