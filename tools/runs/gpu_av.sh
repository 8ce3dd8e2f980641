#!/bin/bash
TAG=${1:-r01av}; OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_faults.py tests/test_gpu_sanitizer.py -q > $OUT/${TAG}_pytest_faults.log 2>&1; echo "exit $?" >> $OUT/${TAG}_pytest_faults.log
timeout 600 ncu --nvtx --nvtx-include "regex:krcv: a3.*/" --metrics gpu__time_duration.sum --clock-control none --csv \
  python -c "
import numpy as np
from paper_conf_ipps_rohlfsz17_b200 import krcv
rng=np.random.default_rng(0); x=rng.uniform(0,1,20000); y=x+rng.normal(0,0.1,x.size)
h=krcv.kr_default_grid(x,200); print(krcv.kr_cv_grid(x,y,h,'epanechnikov')[1])
" > $OUT/${TAG}_ncu_nvtx.csv 2>&1
echo done
