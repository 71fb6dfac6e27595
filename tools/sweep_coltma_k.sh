#!/bin/bash
# coltma units-per-CTA sweep on the 512^3 column cells (G, W, GW) and cfg3 columns
mkdir -p gpurun_out
OUT=gpurun_out/sweep_coltma_${TAG:-x}.jsonl
: > $OUT
for c in cfg5-add-int32-gw cfg5-land-int32-gw cfg5-add-int32-g cfg5-add-int32-w cfg5-add-int64-gw cfg5-add-int64-g cfg3-col; do
  for k in auto 2 4 8 16; do
    if [ $k = auto ]; then E="XR_DUMMY=1"; else E="XR_COLTMA_UNITS_PER_CTA=$k"; fi
    env $E timeout 120 python tools/kdriver.py $c --reps 15 --time | sed "s/^{/{\"k\": \"$k\", /" >> $OUT
  done
done
python - "$OUT" <<'PY'
import json, sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d = json.loads(l)
        print(d["case"], d["k"], round(d["ms_median"] * 1e3, 1), "us", round(d["frac_of_peak"], 3), d["plan"]["splits"], d["plan"]["units"], d["plan"]["grid"])
PY
