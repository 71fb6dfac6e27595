#!/bin/bash
mkdir -p gpurun_out
CASES="cfg5-mul-int32-g cfg5-and-int32-w cfg5-land-int32-gw cfg5-mul-int64-g cfg5-or-int64-w cfg5-mul-fp64-gw"
run() { # label env...
  label=$1; shift
  env "$@" timeout 300 python tools/kdriver.py $CASES --reps 15 --time 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print('$label', d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3), d['plan']['units'], d['plan']['grid'])"
}
run defer-auto XR_X=1
run nodefer-auto XR_LIB_PATH=$PWD/variants/libxreduce_nodefer.so
for gr in 148 222 256 296 342 444; do run grid$gr XR_COLTMA_GRID=$gr; done
for c in 1 2 3; do
  XR_STREAM_CTAS_PER_SM=$c timeout 300 python tools/kdriver.py cfg5-land-fp32-gwv cfg5-mul-fp64-gwv cfg2-f32-sum cfg3-row --reps 15 --time 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print('stream-ctas$c', d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3))"
done
