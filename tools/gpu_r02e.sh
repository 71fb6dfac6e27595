#!/bin/bash
# r02e: colsmall + static one-unit-per-CTA seg -- parity + cfg1 graph latency (vs r01)
mkdir -p gpurun_out
TAG=${TAG:-r02e}
timeout 1200 python -m pytest tests/test_gpu_round2.py tests/test_gpu_parity.py tests/test_gpu_graphs.py tests/test_gpu_multi.py tests/test_gpu_n1.py -q -x > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
timeout 300 python tools/bench_graph.py > gpurun_out/graph_$TAG.jsonl 2>&1
XR_NO_COLSMALL=1 timeout 300 python tools/bench_graph.py > gpurun_out/graph_nocolsmall_$TAG.jsonl 2>&1
XR_NO_PDL=1 timeout 300 python tools/bench_graph.py > gpurun_out/graph_nopdl_$TAG.jsonl 2>&1
timeout 300 python tools/kdriver.py cfg1-g cfg1-w cfg1-v cfg1-gwv --reps 50 --time > gpurun_out/cfg1_$TAG.jsonl 2>&1
tail -3 gpurun_out/pytest_$TAG.log
for f in graph_$TAG graph_nocolsmall_$TAG graph_nopdl_$TAG; do python -c "
import json
for l in open('gpurun_out/$f.jsonl'):
    try: d=json.loads(l)
    except Exception: print(l.strip()[:200]); continue
    print('$f', d['case'], round(d['eager_us_per_call'],2), round(d['graph_us_per_call'],2))"; done
