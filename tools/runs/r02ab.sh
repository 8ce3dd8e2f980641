#!/bin/bash
# r02ab: win_kernel band schedule (every chunk of a band of rows in flight, one chunk per CTA) vs chunk-major: parity, step times, C4 DRAM bytes; ncu of the O(n) build kernels (C2 fused, C4 two-phase and three-phase)
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02ab_build.log 2>&1
KRCV_WIN2_SCHED=band timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_window_variants.py tests/test_gpu_ci.py -m gpu -x -q -p no:cacheprovider > $OUT/r02ab_pytest_band.log 2>&1; echo "exit $?" >> $OUT/r02ab_pytest_band.log
for C in C2 C3 C4 C5; do
  for S in chunk band; do
    KRCV_WIN2_SCHED=$S timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 10 --warmup 3 > $OUT/r02ab_${S}_bench_$C.json 2> /dev/null
  done
done
for S in chunk band; do
  KRCV_WIN2_SCHED=$S timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct --clock-control none -k regex:win_kernel -c 2 --csv --log-file $OUT/r02ab_${S}_C4_dram.csv python bench.py --config C4 --no-alt --no-cpu-baseline --no-extra --steps 1 --warmup 0 > /dev/null 2>&1
done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:pfx_ -c 2 -o $OUT/r02ab_pfx_C2 python bench.py --config C2 --no-alt --no-cpu-baseline --no-extra --steps 1 --warmup 0 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:pfx_ -c 2 -o $OUT/r02ab_pfx_C4 python bench.py --config C4 --no-alt --no-cpu-baseline --no-extra --steps 1 --warmup 0 > /dev/null 2>&1
KRCV_PFX_ITEMS=3 timeout 600 ncu --set full --import-source on --clock-control none -k regex:pfx_ -c 3 -o $OUT/r02ab_pfx3_C4 python bench.py --config C4 --no-alt --no-cpu-baseline --no-extra --steps 1 --warmup 0 > /dev/null 2>&1
echo done
