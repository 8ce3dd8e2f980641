#!/bin/bash
# r02bc: anchors at C2 with the end-of-round kernel (forced KRCV_ANCHORS = 0 / 2 / 4 / 8 / 16), 30 steps each, twice
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02bc
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
for rep in 1 2; do
for J in 0 2 4 8 16; do
  KRCV_ANCHORS=$J timeout 300 python bench.py --config C2 --no-alt --no-cpu-baseline --no-extra --steps 30 --warmup 5 > $OUT/${T}_j${J}_r${rep}_bench_C2.json 2> /dev/null
done
done
echo done
