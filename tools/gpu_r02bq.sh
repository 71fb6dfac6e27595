#!/bin/bash
# r02bq: ncu DRAM % / issue of the round-2 kernels added by the shape-family sweeps
O=gpurun_out/r02bq; mkdir -p $O
KRE='regex:shortrow_kernel|thincol_kernel|rkr_kernel|colflat_kernel|seg_kernel'
M=gpu__time_duration.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,dram__bytes_read.sum,dram__bytes_write.sum,sm__inst_issued.avg.pct_of_peak_sustained_active,launch__grid_size
for c in nest-add-fp32-524288x16x16-v nest-add-fp32-1024x65536x2-v nest-add-fp32-2x65536x1024-g nest-add-fp32-524288x16x16-w nest-add-fp32-64x65536x32-gv nest-add-fp32-8192x273x60-gv nest-add-fp32-5592405x1x24-g nest-add-fp32-1024x65536x2-gw nest-add-fp32-65536x1x2048-v; do
  timeout 300 ncu --metrics $M --clock-control none -k "$KRE" -s 3 -c 1 --csv python tools/kdriver.py $c --reps 1 > $O/$c.csv 2>&1
done
python - <<'PY'
import csv, glob, io, os
rows = []
for f in sorted(glob.glob("gpurun_out/r02bq/*.csv")):
    txt = open(f).read(); i = txt.find('"ID"')
    if i < 0: print(os.path.basename(f), "no data"); continue
    m = {}; kn = ""
    for d in csv.DictReader(io.StringIO(txt[i:])):
        m[d["Metric Name"]] = d["Metric Value"]; kn = d["Kernel Name"]
    rd = float(m["dram__bytes_read.sum"]) if "dram__bytes_read.sum" in m else 0
    print(f"| {os.path.basename(f)[:-4]} | `{kn.split('(')[0]}` | {float(m['gpu__time_duration.sum'])/1e3:.1f} | {m['dram__throughput.avg.pct_of_peak_sustained_elapsed']} | {m['sm__inst_issued.avg.pct_of_peak_sustained_active']} | {m['launch__grid_size']} |")
PY
