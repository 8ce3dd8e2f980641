TAG=r01aq; OUT=gpurun_out; mkdir -p $OUT
timeout 600 python -m pytest tests/test_gpu_property.py tests/test_gpu_window_variants.py -x -q > $OUT/${TAG}_pytest_property.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_property.log
timeout 600 python bench.py > $OUT/${TAG}_bench_C2.json 2> $OUT/${TAG}_bench_C2.err
timeout 600 python bench.py --config C3 --steps 10 --warmup 3 --no-cpu-baseline > $OUT/${TAG}_bench_C3.json 2> $OUT/${TAG}_bench_C3.err
timeout 600 python bench.py --config C1 --steps 20 --warmup 3 --no-cpu-baseline > $OUT/${TAG}_bench_C1.json 2> $OUT/${TAG}_bench_C1.err
