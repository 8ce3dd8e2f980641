#!/bin/bash
# (the sweep_bc_kernel variant this script measured was removed after the run)
# r02af: sweep_bc_kernel (broadcast neighbour streams) parity and A/B vs split / gxg
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02af_build.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_sweep_gxg.py -m gpu -x -q -p no:cacheprovider -k forced > $OUT/r02af_pytest.log 2>&1; echo "exit $?" >> $OUT/r02af_pytest.log
KRCV_SWEEP=bc timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider -k "sweep or algo" > $OUT/r02af_pytest_parity_bc.log 2>&1; echo "exit $?" >> $OUT/r02af_pytest_parity_bc.log
for C in C2 C3 C5 C4; do
  for V in split bc gxg; do
    for G in 4 2; do
      KRCV_SWEEP=$V KRCV_SWEEP_G=$G timeout 300 python bench.py --config $C --algo sweep --no-alt --no-cpu-baseline --no-extra --steps 5 --warmup 3 > $OUT/r02af_${V}${G}_bench_$C.json 2> /dev/null
    done
  done
done
KRCV_SWEEP=bc timeout 600 ncu --set full --import-source on --clock-control none -k regex:sweep_bc -c 1 -o $OUT/r02af_bc_C2 python bench.py --config C2 --algo sweep --no-alt --no-cpu-baseline --no-extra --steps 1 --warmup 0 > /dev/null 2>&1
echo done
