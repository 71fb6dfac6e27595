timeout 900 python -m pytest tests -m "gpu and not slow" -q -x -k "heat" 2>&1 | tail -2
for r in 16 32 64 128; do echo "rows=$r"; XR_HEAT_ROWS=$r timeout 300 python tools/kdriver.py cfg4-heat --reps 21 --time; done
echo "one tile per CTA"; XR_HEAT_ONE_TILE=1 timeout 300 python tools/kdriver.py cfg4-heat --reps 21 --time
