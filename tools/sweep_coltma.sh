for u in 1 2 4 8 16 32; do
  echo "units/cta=$u"; XR_COLTMA_UNITS_PER_CTA=$u python tools/kdriver.py cfg5-xor-int32-gw cfg5-xor-int32-g cfg5-xor-int64-gw --reps 9 --time | python -c "import sys,json; [print('  ',d['case'], round(d['ms_median']*1e3,1), 'us', round(d['frac_of_peak'],3), d['plan']['splits'], d['plan']['units']) for d in map(json.loads, sys.stdin)]"
done
echo "register col kernel"; XR_NO_TMA=1 python tools/kdriver.py cfg5-xor-int32-gw cfg5-xor-int32-g cfg5-xor-int64-gw --reps 9 --time | python -c "import sys,json; [print('  ',d['case'], round(d['ms_median']*1e3,1), 'us', round(d['frac_of_peak'],3), d['plan']['splits'], d['plan']['units']) for d in map(json.loads, sys.stdin)]"
