#!/bin/bash
# after the epilogue warp: re-sweep unit sizes (rkr units/CTA on GV, stream splits on WV, coltma units/CTA on G/GW)
mkdir -p gpurun_out
OUT=gpurun_out/sweep_r01z.jsonl
: > $OUT
run() { env $2 timeout 120 python tools/kdriver.py $1 --reps 25 --time | sed "s/^{/{\"variant\": \"$3\", /" >> $OUT; }
for c in cfg5-mul-int32-gv cfg5-land-fp32-gv cfg5-mul-int64-gv; do
  run $c XR_DUMMY=1 auto
  for k in 6 8 12 16 24; do run $c XR_RKR_UNITS_PER_CTA=$k rkr-k$k; done
done
for c in cfg5-mul-int32-wv cfg5-lor-int32-wv cfg5-mul-int64-wv; do
  run $c XR_DUMMY=1 auto
  for k in 6 8 12 16; do run $c XR_STREAM_SPLITS=$k splits-$k; done
done
for c in cfg5-mul-int32-g cfg5-land-int32-g cfg5-mul-int32-gw cfg5-land-int32-gw cfg5-mul-int64-g; do
  run $c XR_DUMMY=1 auto
  for k in 3 4 5 6; do run $c XR_COLTMA_UNITS_PER_CTA=$k upc-$k; done
done
python - "$OUT" <<'PY'
import json, sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d = json.loads(l)
        print(d["case"], d["variant"], round(d["ms_median"] * 1e3, 1), "us", round(d["ms_min"] * 1e3, 1), round(d["frac_of_peak"], 3), d["plan"]["kernel"], d["plan"]["splits"], d["plan"]["units"], d["plan"].get("grid"))
PY
