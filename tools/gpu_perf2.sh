#!/bin/bash
# quick perf A/B pass: timeline, fixed cost, bench (guided vs not), parity subset
mkdir -p gpurun_out
TAG=${TAG:-perf}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fused.py tests/test_gpu_fullsize.py -q -x -k "parity or fused or cfg2" > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 300 python tools/timeline.py --elements 134217728 268435456 1073741824 --out gpurun_out/timeline_$TAG.jsonl > /dev/null 2>gpurun_out/timeline_$TAG.err
timeout 300 python tools/fixed_cost.py > gpurun_out/fixed_cost_$TAG.jsonl 2>&1
XR_NO_GUIDED=1 timeout 300 python tools/fixed_cost.py > gpurun_out/fixed_cost_noguided_$TAG.jsonl 2>&1
timeout 600 python bench.py --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
XR_NO_GUIDED=1 timeout 600 python bench.py --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_noguided_$TAG.json 2>> gpurun_out/bench_$TAG.err
timeout 600 python tools/kdriver.py cfg5-add-int32-gwv cfg5-mul-fp64-gwv cfg5-land-fp32-gwv nest-add-fp32-1x1x268435456-gwv --reps 15 --time > gpurun_out/shapes_$TAG.jsonl 2>&1
XR_NO_GUIDED=1 timeout 600 python tools/kdriver.py cfg5-add-int32-gwv cfg5-mul-fp64-gwv cfg5-land-fp32-gwv nest-add-fp32-1x1x268435456-gwv --reps 15 --time > gpurun_out/shapes_noguided_$TAG.jsonl 2>&1
tail -3 gpurun_out/pytest_$TAG.log; cut -c1-900 gpurun_out/timeline_$TAG.jsonl
cat gpurun_out/fixed_cost_$TAG.jsonl gpurun_out/fixed_cost_noguided_$TAG.jsonl | grep stream | cut -c1-300
for f in gpurun_out/bench_$TAG.json gpurun_out/bench_noguided_$TAG.json; do python -c "import json; d=json.load(open('$f')); print('$f', d['value'], d['ms_per_step'], d['roofline']['kernel_ms_mean'])"; done
for f in gpurun_out/shapes_$TAG.jsonl gpurun_out/shapes_noguided_$TAG.jsonl; do python -c "
import json,sys
for l in open('$f'):
    try: d=json.loads(l)
    except Exception: continue
    print('$f', d['case'], round(d['ms_median']*1e3,1), round(d['GBps']))"; done
