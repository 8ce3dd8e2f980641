#!/bin/bash
# r02m: algorithm-sized workspace check (parity, host path, distributed, CI tests) + default bench with other_configs
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02m_build.log 2>&1
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_host_path.py tests/test_gpu_distributed.py tests/test_gpu_ci.py tests/test_gpu_ll.py tests/test_gpu_faults.py tests/test_c_consumer.py -m gpu -x -q -p no:cacheprovider > $OUT/r02m_pytest.log 2>&1; echo "exit $?" >> $OUT/r02m_pytest.log
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/r02m_smi.txt 2>&1
timeout 900 python bench.py > $OUT/r02m_bench_default.json 2> $OUT/r02m_bench_default.err
echo done
