#!/bin/bash
# r02af: packed gang tier in the flat column kernel -- parity, cfg1 graph latency, paper gang case A/B
O=gpurun_out/r02af; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_packed.py tests/test_gpu_parity.py tests/test_gpu_graphs.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -2 $O/pytest.log
timeout 300 python tools/bench_graph.py > $O/graph.jsonl 2>&1
XR_NO_PACKED=1 timeout 300 python tools/bench_graph.py > $O/graph_nopacked.jsonl 2>&1
python - <<'PY'
import json
a = [json.loads(l) for l in open("gpurun_out/r02af/graph.jsonl") if l.startswith("{")]
b = {d["case"]: d for d in (json.loads(l) for l in open("gpurun_out/r02af/graph_nopacked.jsonl") if l.startswith("{"))}
for d in a: print(d["case"], "graph us packed", round(d["graph_us_per_call"], 2), "ticket", round(b[d["case"]]["graph_us_per_call"], 2))
PY
timeout 600 python tools/ab_env.py --cases nest-add-int32-1048576x2x32-g nest-add-int32-1048576x2x32-gw nest-add-int32-64x64x128-gw --cfg A: --cfg B:XR_NO_PACKED=1 --rounds 7 --batch 20 2>&1 | tee $O/ab_packed.jsonl
