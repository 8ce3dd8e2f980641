#!/bin/bash
# r02au: factored fast-path bound (KRCV_EFACT) + single-sum accumulation + workspace sized by the anchor count:
# window-variant / anchor / parity tests, C2-C5 A/B against KRCV_EFACT=0
set -u
OUT=gpurun_out; mkdir -p $OUT; T=r02au
CS=paper_conf_ipps_rohlfsz17_b200/csrc
python -c "import __graft_entry__ as g; g.build()" > $OUT/${T}_build.log 2>&1
timeout 1800 python -m pytest tests/test_gpu_window_variants.py tests/test_gpu_anchors.py tests/test_gpu_parity.py -m gpu -x -q -p no:cacheprovider > $OUT/${T}_pytest.log 2>&1; echo "exit $?" >> $OUT/${T}_pytest.log
for V in new old; do
  if [ $V = old ]; then rm -f $CS/build/krcv_device.o; make -s -C $CS EXTRA="-DKRCV_EFACT=0" > $OUT/${T}_build_old.log 2>&1; fi
  for C in C2 C3 C4 C5; do
    timeout 300 python bench.py --config $C --no-alt --no-cpu-baseline --no-extra --steps 20 --warmup 5 > $OUT/${T}_${V}_bench_$C.json 2> /dev/null
  done
done
rm -f $CS/build/krcv_device.o; make -s -C $CS > /dev/null 2>&1
echo done
