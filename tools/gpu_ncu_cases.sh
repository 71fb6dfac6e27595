#!/bin/bash
# usage: TAG=x CASES="regex:case:name ..." bash tools/gpu_ncu_cases.sh
mkdir -p gpurun_out/ncu
for c in $CASES; do
  IFS=: read -r kre case name <<< "$c"
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$kre -s 3 -c 1 -o gpurun_out/ncu/${name}_$TAG -f python tools/kdriver.py $case --reps 1 > gpurun_out/ncu/${name}_$TAG.log 2>&1
  tail -2 gpurun_out/ncu/${name}_$TAG.log
done
