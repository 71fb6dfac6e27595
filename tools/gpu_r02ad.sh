#!/bin/bash
# r02ad: heat loop (32-bit ring counters, hoisted invariants, fmax residual, no per-row proxy fence):
# parity, interleaved process A/B vs the HEAD build (variants/libxreduce_heatold.so), ncu
O=gpurun_out/r02ad; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x -k "heat" > $O/pytest_heat.log 2>&1; echo "pytest rc=$?" >> $O/pytest_heat.log
tail -2 $O/pytest_heat.log
for r in 1 2 3; do
  XR_LIB_PATH=$PWD/variants/libxreduce_heatold.so timeout 300 python tools/heat_ab.py --tag old >> $O/heat_ab.jsonl 2>&1
  timeout 300 python tools/heat_ab.py --tag new >> $O/heat_ab.jsonl 2>&1
done
python - <<'PY'
import json, statistics, collections
d = collections.defaultdict(list)
for l in open("gpurun_out/r02ad/heat_ab.jsonl"):
    if l.startswith("{"):
        x = json.loads(l); d[(x["n"], x["tag"])].append(x)
for n in sorted({k[0] for k in d}):
    row = [n]
    for t in ("old", "new"):
        xs = d[(n, t)]
        ev = statistics.median(x["us_event_median"] for x in xs); bt = statistics.median(x["us_batch_mean"] for x in xs)
        row += [t, ev, bt, round(16 * n * n / bt / 1e3, 1)]
    print(*row)
PY
c=cfg4-heat
timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat_ -s 3 -c 1 -o $O/$c -f python tools/kdriver.py $c --reps 1 > $O/ncu_$c.log 2>&1
ncu -i $O/$c.ncu-rep --page details --csv > $O/${c}_details.csv 2>&1
ncu -i $O/$c.ncu-rep --page source --csv --print-source sass > $O/${c}_sass.csv 2>&1
rm -f $O/$c.ncu-rep
python - <<'PY'
import csv
m = {d["Metric Name"]: d["Metric Value"] for d in csv.DictReader(open("gpurun_out/r02ad/cfg4-heat_details.csv")) if d.get("Metric Name")}
print({k: m.get(k) for k in ("Duration", "DRAM Throughput", "Issue Slots Busy", "Executed Instructions", "Registers Per Thread")})
PY
