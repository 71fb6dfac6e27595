#!/bin/bash
# r02ac: heat sweep with 32-bit ring counters / hoisted invariants -- parity, timings, ncu issue slots
O=gpurun_out/r02ac; mkdir -p $O
timeout 900 python -m pytest tests -m gpu -q -x -k "heat" > $O/pytest_heat.log 2>&1; echo "pytest rc=$?" >> $O/pytest_heat.log
tail -2 $O/pytest_heat.log
for rep in 1 2; do
timeout 600 python tools/kdriver.py cfg4-heat heat-8191 heat-5793 heat-11585 heat-4097 --reps 20 --time 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print(d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3))"
done | tee $O/heat.txt
for c in cfg4-heat heat-8191; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat_ -s 3 -c 1 -o $O/$c -f python tools/kdriver.py $c --reps 1 > $O/ncu_$c.log 2>&1
  ncu -i $O/$c.ncu-rep --page details --csv > $O/${c}_details.csv 2>&1
  ncu -i $O/$c.ncu-rep --page source --csv --print-source sass > $O/${c}_sass.csv 2>&1
  rm -f $O/$c.ncu-rep
done
python - <<'PY'
import csv
for c in ("cfg4-heat", "heat-8191"):
    m = {d["Metric Name"]: d["Metric Value"] for d in csv.DictReader(open(f"gpurun_out/r02ac/{c}_details.csv")) if d.get("Metric Name")}
    print(c, {k: m.get(k) for k in ("Duration", "DRAM Throughput", "Issue Slots Busy", "Executed Instructions", "Registers Per Thread")})
PY
# same-process interleaved A/B of the column box width
timeout 900 python tools/ab_env.py --cases cfg5-mul-fp64-gw cfg5-land-int32-gw cfg5-mul-int64-g cfg5-mul-int32-g cfg5-and-int32-w cfg3-col \
  --cfg A:XR_COLTMA_BOX=1024 --cfg B:XR_COLTMA_BOX=512 --cfg C:XR_COLTMA_BOX=256 --rounds 7 --batch 10 2>&1 | tee $O/ab_box.jsonl
