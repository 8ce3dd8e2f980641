#!/bin/bash
# One gpurun session: tests, smoke, bench, ncu launch list + full capture of the sweep.
# Usage (from the repo root on the GPU box): bash tools/gpu_round.sh [tag] [config]
set -u
TAG=${1:-r01}
CFG=${2:-C2}
OUT=gpurun_out
mkdir -p $OUT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/${TAG}_smi.txt 2>&1
lscpu > $OUT/${TAG}_lscpu.txt 2>&1
nproc >> $OUT/${TAG}_lscpu.txt
timeout 900 python -m pytest tests -m gpu -x -q > $OUT/${TAG}_pytest_gpu.log 2>&1; echo "pytest_gpu exit $?" >> $OUT/${TAG}_pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/${TAG}_smoke.log 2>&1; echo "smoke exit $?" >> $OUT/${TAG}_smoke.log
timeout 600 python bench.py --config $CFG > $OUT/${TAG}_bench_${CFG}.json 2> $OUT/${TAG}_bench_${CFG}.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/${TAG}_launches_${CFG}.csv \
    python bench.py --config $CFG --steps 2 --warmup 1 --no-cpu-baseline > $OUT/${TAG}_ncu_launch_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:sweep_kernel -s 2 -c 1 \
    -o $OUT/${TAG}_sweep_${CFG} -f python bench.py --config $CFG --steps 1 --warmup 2 --no-cpu-baseline > $OUT/${TAG}_ncu_full.log 2>&1
echo done
