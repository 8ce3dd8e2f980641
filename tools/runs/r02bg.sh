#!/bin/bash
# r02bg: final HEAD of round 2 (hist grid slices, min-chunk switch) -- full GPU suite, smoke, default bench
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02bg
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
timeout 3000 python -m pytest tests -m gpu -x -q -p no:cacheprovider > $OUT/${T}_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/${T}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/${T}_smoke.log 2>&1; echo "exit $?" >> $OUT/${T}_smoke.log
timeout 900 python bench.py > $OUT/${T}_bench_default.json 2> $OUT/${T}_bench_default.err
echo done
