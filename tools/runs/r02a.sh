#!/bin/bash
# r02a: FP64 peak microbenchmark + baseline bench lines of HEAD (window kernel r01)
set -u
OUT=gpurun_out; mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/r02a_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02a_build.log 2>&1
timeout 120 python tools/fp64_peak.py --out $OUT/r02a_fp64_peak.json > $OUT/r02a_fp64_peak.log 2>&1
for C in C2 C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --steps 10 --warmup 3 > $OUT/r02a_bench_$C.json 2> $OUT/r02a_bench_$C.err
done
echo done
