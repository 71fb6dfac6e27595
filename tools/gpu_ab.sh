#!/bin/bash
# A/B of the same cells between this tree and another built tree ($AB_DIR), alternating
mkdir -p gpurun_out
OUT=gpurun_out/ab_${TAG:-x}.jsonl
: > $OUT
CELLS=${CELLS:-"cfg5-add-int32-gwv cfg5-lor-fp64-v cfg5-land-fp64-gv cfg5-or-int32-wv cfg5-add-int32-v cfg2-f32-sum"}
for rep in 1 2; do
  for t in new old; do
    if [ $t = new ]; then D=.; else D=$AB_DIR; fi
    for c in $CELLS; do
      timeout 120 python $D/tools/kdriver.py $c --reps 15 --time | sed "s/^{/{\"tree\": \"$t\", \"rep\": $rep, /" >> $OUT
    done
  done
done
python - "$OUT" <<'PY'
import json, sys
for l in open(sys.argv[1]):
    if l.startswith("{"):
        d = json.loads(l)
        print(d["tree"], d["rep"], d["case"], round(d["ms_median"] * 1e3, 1), "us", round(d["frac_of_peak"], 3), d["plan"]["kernel"])
PY
