#!/bin/bash
# && || accumulator as "nonzero" truth (umin / OR folds): parity (full GPU suite) + the logical cfg5 cells
mkdir -p gpurun_out
TAG=${TAG:-logical}

CASES=cfg5-all
timeout 900 python tools/kdriver.py $CASES --reps 15 --time > gpurun_out/cfg5_$TAG.jsonl 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
tail -5 gpurun_out/pytest_gpu_$TAG.log
python - <<PY
import json
rows=[json.loads(l) for l in open('gpurun_out/cfg5_$TAG.jsonl') if l.startswith('{')]
for r in rows: print(r['case'], round(r['ms_median']*1e3,1), round(r['frac_of_peak'],3), r['plan']['kernel'])
PY
cat gpurun_out/bench_$TAG.json
