#!/bin/bash
# r02an/r02ao: anchored fast-path records (anchor_kernel, J = 8 copies): parity suite, A/B against KRCV_ANCHORS=0 and J = 1, 4 at C2-C5
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02an_build.log 2>&1
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_window_variants.py tests/test_gpu_ci.py tests/test_gpu_host_path.py -m gpu -x -q -p no:cacheprovider > $OUT/r02an_pytest.log 2>&1; echo "exit $?" >> $OUT/r02an_pytest.log
for C in C2 C3 C4 C5; do
  for J in def 0 1 4; do
    if [ $J = def ]; then E=""; else E="KRCV_ANCHORS=$J"; fi
    env $E timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02an_j${J}_bench_$C.json 2> $OUT/r02an_j${J}_bench_$C.err
  done
done
timeout 900 python -m pytest tests/test_gpu_sanitizer.py -m gpu -x -q -p no:cacheprovider > $OUT/r02an_sanitizer.log 2>&1; echo "exit $?" >> $OUT/r02an_sanitizer.log
echo done
