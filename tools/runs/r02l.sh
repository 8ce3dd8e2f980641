#!/bin/bash
# r02l: full GPU suite (incl. new CI, gxg, host-path tests, Program-3 C3/C5 golden curves) + smoke
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02l_build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x -p no:cacheprovider --durations=15 > $OUT/r02l_pytest_gpu.log 2>&1; echo "exit $?" >> $OUT/r02l_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/r02l_smoke.log 2>&1; echo "exit $?" >> $OUT/r02l_smoke.log
timeout 900 python -m pytest tests/test_gpu_baseline_curves.py -m gpu -q -s -p no:cacheprovider 2>&1 | grep -E "max rel err" > $OUT/r02l_curves_err.txt
echo done
