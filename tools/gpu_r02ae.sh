#!/bin/bash
# r02ae: issue-slot utilisation of every cfg5 representative kernel (is any other kernel issue bound?)
O=gpurun_out/r02ae; mkdir -p $O
KRE='regex:stream_kernel|seg_kernel|coltma_kernel|col_kernel|colflat_kernel|colsmall_kernel|rows_kernel|rkr_kernel|heat_'
M=gpu__time_duration.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__inst_issued.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,launch__registers_per_thread,launch__grid_size,sm__warps_active.avg.pct_of_peak_sustained_active
for c in cfg2-f32-sum cfg3-col cfg3-row cfg5-mul-int32-g cfg5-and-int32-w cfg5-xor-int32-v cfg5-land-int32-gw cfg5-lor-int32-gv cfg5-mul-fp32-wv cfg5-land-fp32-gwv \
         cfg5-mul-int64-g cfg5-or-int64-w cfg5-xor-int64-v cfg5-mul-fp64-gw cfg5-land-fp64-gv cfg5-lor-fp64-wv cfg5-mul-fp64-gwv; do
  timeout 300 ncu --metrics $M --clock-control none -k "$KRE" -s 3 -c 1 --csv python tools/kdriver.py $c --reps 1 > $O/$c.csv 2>&1
done
python - <<'PY'
import csv, glob, io, os
for f in sorted(glob.glob("gpurun_out/r02ae/*.csv")):
    txt = open(f).read()
    i = txt.find('"ID"')
    if i < 0: print(os.path.basename(f), "no data"); continue
    m = {}
    kn = ""
    for d in csv.DictReader(io.StringIO(txt[i:])):
        m[d["Metric Name"]] = d["Metric Value"]; kn = d["Kernel Name"]
    print(f"{os.path.basename(f)[:-4]:22s} {kn.split('(')[0][:34]:34s} t={m.get('gpu__time_duration.sum')} dram={m.get('dram__throughput.avg.pct_of_peak_sustained_elapsed')} issue={m.get('sm__inst_issued.avg.pct_of_peak_sustained_active')} inst={m.get('smsp__inst_executed.sum')} regs={m.get('launch__registers_per_thread')} warps={m.get('sm__warps_active.avg.pct_of_peak_sustained_active')}")
PY
