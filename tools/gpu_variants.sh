#!/bin/bash
# A/B of library builds (variants/libxreduce_<v>.so, XR_LIB_PATH) on the same cells, alternating
mkdir -p gpurun_out
OUT=gpurun_out/variants_${TAG:-x}.jsonl
: > $OUT
VARS=${VARS:-"p0m1c p1m1 p0m4 p1m3"}
CELLS=${CELLS:-"cfg5-lor-fp64-v cfg5-add-fp64-v cfg5-lor-int64-v cfg5-add-int32-w nest-add-int32-1048576x2x32-g nest-add-fp64-1048576x2x32-g nest-add-fp32-2x1048576x32-w nest-add-int32-4096x1x100-g nest-add-fp32-100000x1x1000-v cfg1-g cfg1-w cfg1-v cfg1-gwv"}
for rep in 1 2; do
  for v in $VARS; do
    XR_LIB_PATH=$PWD/variants/libxreduce_$v.so timeout 300 python tools/kdriver.py $CELLS --reps 15 --time | sed "s/^{/{\"variant\": \"$v\", \"rep\": $rep, /" >> $OUT
  done
done
python - "$OUT" <<'PY'
import json, sys, collections
d = collections.defaultdict(dict)
for l in open(sys.argv[1]):
    if l.startswith("{"):
        r = json.loads(l)
        d[r["case"]].setdefault(r["variant"], []).append(r["ms_median"] * 1e3)
for c, v in d.items():
    print(c, "  ".join(f"{k}={min(x):.1f}" for k, x in v.items()))
PY
