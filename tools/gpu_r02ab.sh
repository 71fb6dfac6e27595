#!/bin/bash
# r02ab: per-shape TMA box width -- parity (column shapes, full sizes) + cfg5 / cfg3 timings
O=gpurun_out/r02ab; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_round2.py tests/test_gpu_graphs.py tests/test_sass.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -2 $O/pytest.log
timeout 900 python tools/kdriver.py cfg5-all --reps 9 --time > $O/cfg5.jsonl 2>&1
timeout 600 python tools/kdriver.py cfg3-col cfg3-row cfg2-f32-sum --reps 20 --time > $O/shapes.jsonl 2>&1
python - <<'PY'
import json
old = {json.loads(l)["case"]: json.loads(l) for l in open("profiles/cfg5_r02w.jsonl") if l.startswith("{")}
rows = []
for l in open("gpurun_out/r02ab/cfg5.jsonl"):
    if not l.startswith("{"): continue
    d = json.loads(l); o = old.get(d["case"])
    if o and d["case"].split("-")[-1] in ("g", "w", "gw"):
        rows.append((d["case"], round(o["ms_median"]*1e3, 1), round(d["ms_median"]*1e3, 1)))
for r in rows: print(*r)
import statistics
print("median ratio new/old", statistics.median(n/o for _, o, n in rows))
for l in open("gpurun_out/r02ab/shapes.jsonl"):
    if l.startswith("{"): d = json.loads(l); print(d["case"], round(d["ms_median"]*1e3, 1), round(d["frac_of_peak"], 3))
PY
