#!/bin/bash
# guided-unit A/B: default (2-stage min, 2-deep claims) vs 1-stage / 4-stage min vs equal units
mkdir -p gpurun_out
TAG=${TAG:-perf3}
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -k "cfg2 or staged or fuzz" > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
for v in "default:" "min16k:XR_GUIDED_MIN_BYTES=16384" "min64k:XR_GUIDED_MIN_BYTES=65536" "equal:XR_NO_GUIDED=1"; do
  name=${v%%:*}; envs=${v#*:}
  env $envs timeout 300 python tools/fixed_cost.py 2>&1 | grep stream | sed "s/^/$name /" >> gpurun_out/fc_$TAG.txt
  env $envs timeout 300 python tools/kdriver.py cfg5-add-int32-gwv cfg5-mul-fp64-gwv --reps 15 --time 2>&1 | sed "s/^/$name /" >> gpurun_out/k_$TAG.txt
done
tail -2 gpurun_out/pytest_$TAG.log
cut -c1-330 gpurun_out/fc_$TAG.txt
python - <<'PY'
import json
for l in open("gpurun_out/k_perf3.txt" if False else "gpurun_out/k_${TAG}.txt".replace("${TAG}", __import__("os").environ.get("TAG","perf3"))):
    name, js = l.split(" ", 1)
    try: d = json.loads(js)
    except Exception: continue
    print(name, d["case"], round(d["ms_median"]*1e3, 1), round(d["GBps"]))
PY
