#!/bin/bash
# r02e: smem task accumulators, 32-bit record index math; MINB sweep 6/7/8 (8 default)
set -u
OUT=gpurun_out; mkdir -p $OUT
CS=paper_conf_ipps_rohlfsz17_b200/csrc
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02e_build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window_variants.py -m gpu -x -q > $OUT/r02e_pytest.log 2>&1; echo "exit $?" >> $OUT/r02e_pytest.log
for C in C2 C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --steps 10 --warmup 3 > $OUT/r02e_bench_$C.json 2> $OUT/r02e_bench_$C.err
done
for MB in 6 7; do
  rm -f $CS/build/krcv_device.o; make -s -C $CS EXTRA=-DKRCV_WIN2_MINB=$MB > $OUT/r02e_build_mb$MB.log 2>&1
  for C in C2 C4 C5; do
    timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --steps 10 --warmup 3 > $OUT/r02e_mb${MB}_bench_$C.json 2> $OUT/r02e_mb${MB}_bench_$C.err
  done
done
rm -f $CS/build/krcv_device.o; make -s -C $CS > /dev/null 2>&1
echo done
