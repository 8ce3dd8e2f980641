#!/bin/bash
# bash tools/tune2.sh TAG "V:G V:G ..." CFG...
OUT=gpurun_out; mkdir -p $OUT; TAG=$1; shift; VGS=$1; shift; CFGS=${@:-C2}
for VG in $VGS; do V=${VG%%:*}; G=${VG##*:}
  KRCV_SWEEP=$V KRCV_SWEEP_G=$G timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "small or dyadic or emulation or worked or guard or duplicate or user_grid or C1 or C2_seed0" > $OUT/${TAG}_pytest_${V}_G$G.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_${V}_G$G.log
done
for C in $CFGS; do for VG in $VGS; do V=${VG%%:*}; G=${VG##*:}
  KRCV_SWEEP=$V KRCV_SWEEP_G=$G timeout 300 python bench.py --config $C --steps ${STEPS:-5} --warmup ${WARM:-2} --no-cpu-baseline > $OUT/${TAG}_${C}_${V}_G$G.json 2>$OUT/${TAG}_${C}_${V}_G$G.err
done; done
echo done
