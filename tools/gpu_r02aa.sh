#!/bin/bash
# r02aa: column TMA kernel box width A/B (1024 / 512 / 256 B) on the cfg5 column cells and cfg3 columns
O=gpurun_out/r02aa; mkdir -p $O
XR_COLTMA_BOX=256 XR_SMALL_BYTES=0 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "col or every or mask or ragged" > $O/pytest256.log 2>&1; echo "pytest rc=$?" >> $O/pytest256.log
tail -2 $O/pytest256.log
sw() {
  local spec=$1; shift
  for c in "$@"; do
    env $spec timeout 300 python tools/kdriver.py $c --reps 15 --time 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print('$spec', d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3))"
  done
}
for rep in 1 2; do
for b in 1024 512 256; do
  sw XR_COLTMA_BOX=$b cfg5-mul-int64-g cfg5-or-int64-w cfg5-mul-fp64-gw cfg5-mul-int32-g cfg5-and-int32-w cfg5-land-int32-gw cfg3-col
done
done | tee $O/box.txt
for b in 1024 256; do
  XR_COLTMA_BOX=$b timeout 300 python tools/timeline.py --nest 512 512 512 --mask g --dtype fp64 --reps 10 >> $O/timeline.jsonl 2>&1
  XR_COLTMA_BOX=$b timeout 300 python tools/timeline.py --nest 512 512 512 --mask g --dtype fp32 --reps 10 >> $O/timeline.jsonl 2>&1
done
python - <<'PY'
import json
for l in open("gpurun_out/r02aa/timeline.jsonl"):
    try: d = json.loads(l)
    except Exception: continue
    print(d["dtype"], d["mask"], d["plan"], "ev", round(d["event_ms_median"]*1e3,1), "cons_end", d.get("cons_end_us"), "claim_last", d.get("last_real_claim_us"), "unit_us", d.get("unit_us"))
PY
