#!/bin/bash
mkdir -p gpurun_out
for k in 4 8 16 32; do
  XR_MULTI_UNITS_PER_CTA=$k timeout 300 python tools/bench_multi.py 2>&1 | grep "16777216\|256, 256" | python -c "
import sys,json
for l in sys.stdin:
    d=json.loads(l); print('upc=$k', d['dims'], round(d['multi_ms']*1e3,1), round(d['multi_GBps']))"
done
