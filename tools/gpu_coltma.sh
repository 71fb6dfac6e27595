#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-coltma}
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_round2.py -q -x > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
tail -3 gpurun_out/pytest_$TAG.log
CASES="cfg5-mul-int32-g cfg5-and-int32-w cfg5-land-int32-gw cfg5-mul-int64-g cfg5-or-int64-w cfg5-mul-fp64-gw cfg3-col"
for k in auto 2 4 8 16; do
  if [ $k = auto ]; then E=""; else E="XR_COLTMA_UNITS_PER_CTA=$k"; fi
  env $E timeout 300 python tools/kdriver.py $CASES --reps 15 --time 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print('k=$k', d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3), d['plan']['units'], d['plan']['splits'])"
done
