#!/bin/bash
O=gpurun_out/r02bi; mkdir -p $O
timeout 1500 python tools/ab_env.py --cases cfg5-xor-int64-v cfg5-lor-int32-gv cfg5-land-fp64-gv cfg5-mul-int64-gv nest-add-fp32-131072x1x1024-v nest-add-fp32-32768x1x4096-v nest-add-fp32-8192x1x8191-v \
  --cfg A: --cfg w8_4k:XR_SEG_W8_MAX=4096 --rounds 5 --batch 10 2>&1 | tee $O/ab_seg_w8_pow2.jsonl
XR_SEG_W8_MAX=4096 timeout 300 python tools/bench_graph.py > $O/graph_w8.jsonl 2>&1
timeout 300 python tools/bench_graph.py > $O/graph_a.jsonl 2>&1
python - <<'PY'
import json
a = {json.loads(l)["case"]: json.loads(l) for l in open("gpurun_out/r02bi/graph_a.jsonl") if l.startswith("{")}
b = {json.loads(l)["case"]: json.loads(l) for l in open("gpurun_out/r02bi/graph_w8.jsonl") if l.startswith("{")}
for k in a: print(k, round(a[k]["graph_us_per_call"], 2), round(b[k]["graph_us_per_call"], 2))
PY
