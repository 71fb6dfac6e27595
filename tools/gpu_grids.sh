#!/bin/bash
mkdir -p gpurun_out
run() { label=$1; cases=$2; shift 2
  env "$@" timeout 300 python tools/kdriver.py $cases --reps 15 --time 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print('$label', d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3), d['plan']['grid'])"
}
C="cfg5-mul-int32-g cfg5-and-int32-w cfg5-land-int32-gw cfg5-mul-int64-g cfg5-or-int64-w cfg5-mul-fp64-gw cfg3-col"
run coltma-auto "$C" XR_X=1
for gr in 222 256 296 342 444; do run coltma-grid$gr "$C" XR_COLTMA_GRID=$gr; done
R="cfg5-lor-int32-gv cfg5-mul-fp32-gv cfg5-land-fp32-gv"
run rkr-auto "$R" XR_X=1
for gr in 222 296 444; do run rkr-grid$gr "$R" XR_RKR_GRID=$gr; done
V="cfg5-xor-int32-v cfg5-mul-fp32-v"
run rows-auto "$V" XR_X=1
for gr in 222 296 444; do run rows-grid$gr "$V" XR_ROWS_GRID=$gr; done
S="cfg2-f32-sum cfg5-mul-fp64-gwv cfg5-land-fp64-gv cfg5-mul-fp32-wv nest-add-fp32-134217728x1x1-gwv"
run stream-2sm "$S" XR_X=1
run stream-3sm "$S" XR_STREAM_CTAS_PER_SM=3
