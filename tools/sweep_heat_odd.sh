#!/bin/bash
# tile-row sweep of the odd-width persistent heat kernel (XR_HEAT_ROWS)
mkdir -p gpurun_out
for r in 6 8 12 16 24 32; do
  XR_HEAT_ROWS=$r timeout 300 python tools/kdriver.py heat-8191 heat-5793 heat-11585 --reps 15 --time 2>&1 | python -c "
import sys, json
for l in sys.stdin:
    if l.startswith('{'):
        d = json.loads(l); print('rows=$r', d['case'], round(d['ms_median'] * 1e3, 1), round(d['frac_of_peak'], 3))
"
done > gpurun_out/sweep_heat_odd.txt
cat gpurun_out/sweep_heat_odd.txt
