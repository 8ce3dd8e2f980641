#!/bin/bash
# tuning sweep: parity per variant/G + bench per variant/G for given configs
OUT=gpurun_out; mkdir -p $OUT; TAG=${1:-tune}; shift
CFGS=${@:-C2}
for V in gxg split; do for G in 1 2 4; do
  KRCV_SWEEP=$V KRCV_SWEEP_G=$G timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "small or dyadic or emulation or worked or guard or duplicate" > $OUT/${TAG}_pytest_${V}_G$G.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_${V}_G$G.log
done; done
for C in $CFGS; do for V in gxg split; do for G in 1 2 4; do
  KRCV_SWEEP=$V KRCV_SWEEP_G=$G timeout 300 python bench.py --config $C --steps 10 --warmup 3 --no-cpu-baseline > $OUT/${TAG}_${C}_${V}_G$G.json 2>$OUT/${TAG}_${C}_${V}_G$G.err
done; done; done
echo done
