#!/bin/bash
# r02bb: histogram path in grid slices for m beyond one shared-memory histogram: hist tests; C2 hist bench
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02bb
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_hist.py tests/test_gpu_faults.py tests/test_gpu_host_path.py -m gpu -x -q -p no:cacheprovider > $OUT/${T}_pytest.log 2>&1; echo "exit $?" >> $OUT/${T}_pytest.log
KRCV_ALGO=hist timeout 300 python bench.py --config C2 --no-alt --no-cpu-baseline --no-extra --steps 3 --warmup 3 > $OUT/${T}_hist_bench_C2.json 2> $OUT/${T}_hist_bench_C2.err
timeout 300 python bench.py --config C2 --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/${T}_bench_C2.json 2> /dev/null
echo done
