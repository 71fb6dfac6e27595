#!/bin/bash
mkdir -p gpurun_out
TAG=${TAG:-r02h}
timeout 1200 python -m pytest tests/test_gpu_round2.py tests/test_gpu_parity.py tests/test_gpu_fused.py tests/test_gpu_graphs.py -q -x > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 300 python tools/bench_graph.py > gpurun_out/graph_$TAG.jsonl 2>&1
XR_NO_CLUSTER=1 timeout 300 python tools/bench_graph.py > gpurun_out/graph_nocluster_$TAG.jsonl 2>&1
tail -4 gpurun_out/pytest_$TAG.log
for f in graph_$TAG graph_nocluster_$TAG; do python -c "
import json
for l in open('gpurun_out/$f.jsonl'):
    try: d=json.loads(l)
    except Exception: print(l.strip()[:300]); continue
    print('$f', d['case'], round(d['eager_us_per_call'],2), round(d['graph_us_per_call'],2))"; done
