timeout 900 python -m pytest tests -m "gpu and not slow" -q -x 2>&1 | tail -2
for u in 2 4 8 16; do
  echo "units/cta=$u"; XR_COLTMA_UNITS_PER_CTA=$u timeout 300 python tools/kdriver.py cfg5-xor-int32-gw cfg5-xor-int32-g cfg5-xor-int32-w cfg5-xor-int64-gw cfg3-col --reps 9 --time | python -c "import sys,json; [print('  ',d['case'], round(d['ms_median']*1e3,1), 'us', round(d['frac_of_peak'],3), d['plan']['splits'], d['plan']['units']) for d in map(json.loads, sys.stdin)]"
done
timeout 300 python tools/kdriver.py cfg2-f32-sum cfg2-i64-sum cfg3-row cfg5-xor-int32-gwv cfg5-xor-int32-wv --reps 15 --time | python -c "import sys,json; [print('  ',d['case'], round(d['ms_median']*1e3,1), 'us', round(d['frac_of_peak'],3), d['plan']['splits'], d['plan']['units']) for d in map(json.loads, sys.stdin)]"
