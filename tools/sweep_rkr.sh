#!/bin/bash
# RKR (cfg5 GV) stream-vs-seg and split sweep; rows-kernel units sweep (cfg5 V)
mkdir -p gpurun_out
OUT=gpurun_out/sweep_rkr_${TAG:-x}.jsonl
: > $OUT
CASES="cfg5-add-int32-gv cfg5-lor-int32-gv cfg5-land-fp32-gv cfg5-add-fp32-gv cfg5-add-int64-gv cfg5-land-fp64-gv"
for c in $CASES; do
  XR_NO_RKR_STREAM=1 timeout 120 python tools/kdriver.py $c --reps 15 --time | sed 's/^{/{"variant": "seg", /' >> $OUT
  for s in auto 2 4 8 16 32; do
    if [ $s = auto ]; then E="XR_DUMMY=1"; else E="XR_STREAM_SPLITS=$s"; fi
    env $E timeout 120 python tools/kdriver.py $c --reps 15 --time | sed "s/^{/{\"variant\": \"stream-$s\", /" >> $OUT
  done
done
for c in cfg5-add-int32-v cfg5-mul-int32-v cfg5-land-fp32-v; do
  for k in 2 4 8 16 32; do
    XR_ROWS_UNITS_PER_CTA=$k timeout 120 python tools/kdriver.py $c --reps 15 --time | sed "s/^{/{\"variant\": \"rows-k$k\", /" >> $OUT
  done
done
python - "$OUT" <<'PY'
import json, sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d = json.loads(l)
        print(d["case"], d["variant"], round(d["ms_median"] * 1e3, 1), "us", round(d["frac_of_peak"], 3), d["plan"]["kernel"], d["plan"]["splits"], d["plan"]["units"])
PY
