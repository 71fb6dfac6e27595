#!/bin/bash
mkdir -p gpurun_out
CASES="nest-add-fp32-134217728x1x1-gwv nest-add-fp32-268435456x1x1-gwv cfg2-f32-sum cfg3-row cfg5-mul-fp32-wv cfg5-mul-fp64-gwv cfg5-land-fp64-gv"
run() { label=$1; shift
  env "$@" timeout 300 python tools/kdriver.py $CASES --reps 21 --time 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print('$label', d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3), d['plan']['units'])"
}
for rep in 1 2; do
run ns4-3sm XR_X=1
run ns4-2sm XR_STREAM_CTAS_PER_SM=2
run ns6 XR_LIB_PATH=$PWD/variants/libxreduce_ns6.so
run ns8 XR_LIB_PATH=$PWD/variants/libxreduce_ns8.so
done
