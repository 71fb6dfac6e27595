#!/bin/bash
# r02al: group size of the two-level column gang tier (64 / 32 / 16 unit partials per group) x units per CTA
O=gpurun_out/r02al; mkdir -p $O
for r in 1 2 3; do
  for g in 64 32 16; do
    if [ $g = 64 ]; then unset XR_LIB_PATH; else export XR_LIB_PATH=$PWD/variants/libxreduce_g$g.so; fi
    timeout 600 python tools/ab_env.py --cases cfg5-land-int32-gw cfg5-mul-fp32-gw cfg5-mul-fp64-gw cfg3-col \
      --cfg A: --cfg k4:XR_COLTMA_UNITS_PER_CTA=4 --cfg k8:XR_COLTMA_UNITS_PER_CTA=8 --rounds 3 --batch 10 2>&1 | sed "s/^{/{\"group\": $g, \"rep\": $r, /" >> $O/ab_group.jsonl
  done
done
unset XR_LIB_PATH
python - <<'PY'
import json, statistics, collections
d = collections.defaultdict(list)
for l in open("gpurun_out/r02al/ab_group.jsonl"):
    if l.startswith("{"):
        x = json.loads(l); d[(x["case"], x["cfg"], x["group"])].append(x["us_median"])
for k in sorted(d): print(*k, round(statistics.median(d[k]), 2), d[k])
PY
