#!/bin/bash
# odd-width heat grids through the persistent bulk kernel (per-row 8-B staging shift): parity + timing vs the register sweep
mkdir -p gpurun_out
TAG=${TAG:-heatodd}
timeout 900 python -m pytest tests -m gpu -q -x -k "heat" > gpurun_out/pytest_heat_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_heat_$TAG.log
tail -3 gpurun_out/pytest_heat_$TAG.log
timeout 600 python tools/kdriver.py cfg4-heat heat-8191 heat-5793 heat-11585 --reps 20 --time > gpurun_out/heat_$TAG.jsonl 2>&1
XR_NO_ODD_BULK=1 timeout 600 python tools/kdriver.py heat-8191 heat-5793 heat-11585 --reps 20 --time > gpurun_out/heat_reg_$TAG.jsonl 2>&1
cat gpurun_out/heat_$TAG.jsonl gpurun_out/heat_reg_$TAG.jsonl | cut -c1-220
