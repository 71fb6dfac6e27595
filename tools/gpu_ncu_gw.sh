#!/bin/bash
# ncu --set full of the remaining-gap ring cells (512^3 32-bit GW coltma, GV rkr) at HEAD
mkdir -p gpurun_out/ncu
TAG=${TAG:-gw}
TAG=$TAG CASES="coltma:cfg5-land-int32-gw:gwland coltma:cfg5-add-int32-gw:gwadd rkr:cfg5-add-int32-gv:gvadd coltma:cfg5-add-int32-g:gadd" bash tools/gpu_ncu_cases.sh
for n in gwland gwadd gvadd gadd; do
  ncu -i gpurun_out/ncu/${n}_$TAG.ncu-rep --page raw --csv --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,launch__registers_per_thread > gpurun_out/ncu/${n}_$TAG.csv 2>&1
  tail -1 gpurun_out/ncu/${n}_$TAG.csv
done
