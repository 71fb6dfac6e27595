#!/bin/bash
# r02g: transform-reduce bulk ring, overlapped sharded heat, multi-kernel register cap
mkdir -p gpurun_out
TAG=${TAG:-r02g}
timeout 1200 python -m pytest tests/test_gpu_round2.py tests/test_gpu_nccl1.py tests/test_gpu_n1.py tests/test_gpu_multi.py -q -x > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 300 python tools/kdriver.py mc-pi-27 mc-pi-28 mc-pi-29 dot-rows --reps 15 --time > gpurun_out/xform_$TAG.jsonl 2>&1
XR_NO_XF_STREAM=1 timeout 300 python tools/kdriver.py mc-pi-27 mc-pi-28 mc-pi-29 dot-rows --reps 15 --time > gpurun_out/xform_reg_$TAG.jsonl 2>&1
timeout 300 python tools/bench_multi.py > gpurun_out/multi_$TAG.jsonl 2>&1
XR_LIB_PATH=$PWD/variants/libxreduce_multiminb1.so timeout 300 python tools/bench_multi.py > gpurun_out/multi_minb1_$TAG.jsonl 2>&1
tail -3 gpurun_out/pytest_$TAG.log
for f in xform_$TAG xform_reg_$TAG; do python -c "
import json
for l in open('gpurun_out/$f.jsonl'):
    try: d=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print('$f', d['case'], round(d['ms_median']*1e3,1), round(d['GBps']), round(d['frac_of_peak'],3))"; done
cut -c1-250 gpurun_out/multi_$TAG.jsonl; cut -c1-250 gpurun_out/multi_minb1_$TAG.jsonl
