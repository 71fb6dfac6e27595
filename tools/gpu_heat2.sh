#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-heat2}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_nccl1.py tests/test_gpu_fullsize.py -q -x -k "heat" > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 600 python tools/kdriver.py cfg4-heat heat-8191 heat-5793 heat-11585 heat-4097 --reps 15 --time > gpurun_out/heat_$TAG.jsonl 2>&1
tail -3 gpurun_out/pytest_$TAG.log
python -c "
import json
for l in open('gpurun_out/heat_$TAG.jsonl'):
    try: d=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print(d['case'], round(d['ms_median']*1e3,1), round(d['GBps']), round(d['frac_of_peak'],3))"
