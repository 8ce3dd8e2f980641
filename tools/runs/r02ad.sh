#!/bin/bash
# r02ad: fused build with one warp scan (terms kept across the grid barrier) + two-level merge-path bucket-table fill; parity, sanitizer, step times, ncu of both kernels
set -u
OUT=gpurun_out; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.build()" > $OUT/r02ad_build.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_baseline_curves.py tests/test_gpu_window_variants.py tests/test_gpu_ci.py tests/test_gpu_property.py tests/test_gpu_sanitizer.py tests/test_gpu_host_path.py -m gpu -x -q -p no:cacheprovider > $OUT/r02ad_pytest.log 2>&1; echo "exit $?" >> $OUT/r02ad_pytest.log
for C in C1 C2 C3 C4 C5; do
  timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/r02ad_bench_$C.json 2> /dev/null
done
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"pfx_fused|bkt_fill" -c 2 -o $OUT/r02ad_build_C2 python bench.py --config C2 --no-alt --no-cpu-baseline --no-extra --steps 1 --warmup 0 > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"bkt_fill" -c 1 -o $OUT/r02ad_bkt_C5 python bench.py --config C5 --no-alt --no-cpu-baseline --no-extra --steps 1 --warmup 0 > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02ad_launches_C5.csv python bench.py --config C5 --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > /dev/null 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/r02ad_launches_C2.csv python bench.py --config C2 --steps 2 --warmup 1 --no-alt --no-cpu-baseline --no-extra > /dev/null 2>&1
echo done
