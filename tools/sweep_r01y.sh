#!/bin/bash
# Weak cfg5 cells (32-bit, 512 MiB, per-output gang tier): WV stream splits, G/GW coltma units per CTA
mkdir -p gpurun_out
OUT=gpurun_out/sweep_r01y.jsonl
: > $OUT
for c in cfg5-mul-int32-wv cfg5-lor-int32-wv cfg5-land-fp32-wv; do
  for s in auto 4 8 12 16 32 64; do
    if [ $s = auto ]; then E="XR_DUMMY=1"; else E="XR_STREAM_SPLITS=$s"; fi
    env $E timeout 120 python tools/kdriver.py $c --reps 25 --time | sed "s/^{/{\"variant\": \"splits-$s\", /" >> $OUT
  done
done
for c in cfg5-mul-int32-g cfg5-lor-int32-g cfg5-mul-int32-gw cfg5-lor-int32-gw cfg5-mul-int32-w; do
  for k in auto 1 2 3 4 6 8; do
    if [ $k = auto ]; then E="XR_DUMMY=1"; else E="XR_COLTMA_UNITS_PER_CTA=$k"; fi
    env $E timeout 120 python tools/kdriver.py $c --reps 25 --time | sed "s/^{/{\"variant\": \"upc-$k\", /" >> $OUT
  done
done
python - "$OUT" <<'PY'
import json, sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d = json.loads(l)
        print(d["case"], d["variant"], round(d["ms_median"] * 1e3, 1), "us", round(d["ms_min"] * 1e3, 1), round(d["frac_of_peak"], 3), d["plan"]["kernel"], d["plan"]["splits"], d["plan"]["units"], d["plan"].get("grid"))
PY
