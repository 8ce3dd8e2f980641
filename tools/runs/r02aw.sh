#!/bin/bash
# r02aw: up to 16 anchored copies (kAncMax 16; the rule now picks 16 at C3): anchor tests incl. J = 16,
# C3 / C5 A/B J = 16 vs 8, C4 default
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02aw
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_anchors.py -m gpu -x -q -p no:cacheprovider > $OUT/${T}_pytest.log 2>&1; echo "exit $?" >> $OUT/${T}_pytest.log
for C in C3 C5; do
  for J in 16 8; do
    KRCV_ANCHORS=$J timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/${T}_j${J}_bench_$C.json 2> /dev/null
  done
done
timeout 300 python bench.py --config C4 --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/${T}_jdef_bench_C4.json 2> /dev/null
echo done
