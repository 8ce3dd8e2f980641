#!/bin/bash
# r02az: Epanechnikov rows keep fl(x_r - o) instead of the dd shift (the dd path recomputes it; KRCV_ROW_DLA): tests + C2-C5 benches
# parity tests; C2-C5 benches (compare r02ax / r02av)
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02az
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_window_variants.py tests/test_gpu_anchors.py tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider > $OUT/${T}_pytest.log 2>&1; echo "exit $?" >> $OUT/${T}_pytest.log
for C in C2 C3 C4 C5 C2; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 30 --warmup 5 > $OUT/${T}_bench_$C.json 2> /dev/null
done
echo done
