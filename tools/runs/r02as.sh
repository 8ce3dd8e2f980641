#!/bin/bash
# r02as: a shard builds only its rows' anchored copies (task anchors clamped to them); anchor + parity + distributed
# tests; default bench (C3-C5 projections with per-shard build times); C4 J = 2 / 4 / 8 A/B
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02as
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_anchors.py tests/test_gpu_parity.py tests/test_gpu_distributed.py tests/test_gpu_baseline_curves.py -m gpu -x -q -p no:cacheprovider > $OUT/${T}_pytest.log 2>&1; echo "exit $?" >> $OUT/${T}_pytest.log
timeout 900 python bench.py > $OUT/${T}_bench_default.json 2> $OUT/${T}_bench_default.err
for J in 2 4 8; do
  KRCV_ANCHORS=$J timeout 300 python bench.py --config C4 --no-alt --no-cpu-baseline --no-extra --steps 5 --warmup 3 > $OUT/${T}_j${J}_bench_C4.json 2> /dev/null
done
echo done
