#!/bin/bash
mkdir -p gpurun_out
for v in default acqrel; do
  if [ $v = default ]; then L=""; else L="XR_LIB_PATH=$PWD/variants/libxreduce_$v.so"; fi
  env $L timeout 300 python tools/bench_graph.py 2>&1 | sed "s/^/$v /" >> gpurun_out/graph_acqrel.txt
  env $L timeout 300 python tools/kdriver.py cfg5-mul-int32-gw cfg5-lor-int32-gv cfg5-mul-fp32-wv cfg5-land-fp32-gwv cfg2-f32-sum --reps 15 --time 2>&1 | sed "s/^/$v /" >> gpurun_out/k_acqrel.txt
done
cat gpurun_out/graph_acqrel.txt | python -c "
import sys,json
for l in sys.stdin:
    v,js=l.split(' ',1)
    try: d=json.loads(js)
    except Exception: continue
    print(v, d['case'], round(d['graph_us_per_call'],2))"
cat gpurun_out/k_acqrel.txt | python -c "
import sys,json
for l in sys.stdin:
    v,js=l.split(' ',1)
    try: d=json.loads(js)
    except Exception: continue
    print(v, d['case'], round(d['ms_median']*1e3,1))"
