#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-multi2}
timeout 1200 python -m pytest tests/test_gpu_round2.py tests/test_gpu_multi.py -q -x > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 300 python tools/bench_multi.py > gpurun_out/multi_$TAG.jsonl 2>&1
XR_NO_MULTI_STREAM=1 timeout 300 python tools/bench_multi.py > gpurun_out/multi_reg_$TAG.jsonl 2>&1
tail -15 gpurun_out/pytest_$TAG.log | grep -v "^$"
for f in multi_$TAG multi_reg_$TAG; do python -c "
import json
for l in open('gpurun_out/$f.jsonl'):
    try: d=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print('$f', d['dims'], d['levels'] if isinstance(d['levels'], str) else 'mixed', round(d['multi_ms']*1e3,1), round(d['multi_GBps']), round(d['speedup'],2))"; done
