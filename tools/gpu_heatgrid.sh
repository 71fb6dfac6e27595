#!/bin/bash
for c in 1 2 3 4 5 6 8; do
  for rows in 8 12 16; do
  XR_HEAT_CTAS_PER_SM=$c XR_HEAT_ROWS=$rows timeout 300 python tools/kdriver.py cfg4-heat heat-8191 --reps 15 --time 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print('ctas$c rows$rows', d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3))"
  done
done
