#!/bin/bash
# r02y: column TMA kernel unit size x deferred group tickets (variants/libxreduce_defer.so)
O=gpurun_out/r02y; mkdir -p $O
for lib in default defer; do
  if [ $lib = defer ]; then export XR_LIB_PATH=$PWD/variants/libxreduce_defer.so; else unset XR_LIB_PATH; fi
  for k in 2 4 8 16 32 64; do
    for c in cfg5-mul-int64-g cfg5-mul-fp64-gw cfg5-mul-int32-g cfg5-land-int32-gw; do
      XR_COLTMA_UNITS_PER_CTA=$k timeout 300 python tools/kdriver.py $c --reps 15 --time 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print('$lib k$k', d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3))"
    done
  done
done | tee $O/coltma_units_defer.txt
