#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-cfg5}
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 900 python tools/kdriver.py cfg5-all --reps 9 --time > gpurun_out/cfg5_$TAG.jsonl 2>&1
timeout 600 python bench.py --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
tail -2 gpurun_out/pytest_$TAG.log
python - <<PY
import json, statistics
fr=[]; by={}
for l in open("gpurun_out/cfg5_$TAG.jsonl"):
    try: d=json.loads(l)
    except Exception: continue
    fr.append(d["frac_of_peak"]); k=d["case"].split("-")[-1]+("64" if d["dtype"] in ("int64","fp64") else "32")
    by.setdefault(k,[]).append(d["ms_median"]*1e3)
print(len(fr), round(min(fr),3), round(statistics.median(fr),3), round(max(fr),3))
for k,v in sorted(by.items()): print(k, round(min(v),1), round(statistics.median(v),1), round(max(v),1))
d=json.load(open("gpurun_out/bench_$TAG.json")); print(d["value"], d["ms_per_step"], d["roofline"]["kernel"])
PY
