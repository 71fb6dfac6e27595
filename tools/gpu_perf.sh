#!/bin/bash
# GPU pass: parity tests (fast subset unless FULL=1), per-shape timings, bench line
mkdir -p gpurun_out
TAG=${TAG:-perf}
if [ "${FULL:-0}" = "1" ]; then SEL="gpu"; else SEL="gpu and not slow"; fi
timeout 2400 python -m pytest tests -m "$SEL" -q -x > gpurun_out/pytest_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_$TAG.log
tail -4 gpurun_out/pytest_$TAG.log
timeout 600 python tools/kdriver.py cfg2-f32-sum cfg2-f32-max cfg2-f32-min cfg2-i64-sum cfg2-i64-max cfg2-i64-min cfg2-f64-sum cfg3-row cfg3-col cfg4-heat cfg1-g cfg1-w cfg1-v cfg1-gwv --reps 20 --time > gpurun_out/shapes_$TAG.jsonl 2>&1
timeout 900 python tools/kdriver.py cfg5-all --reps 7 --time > gpurun_out/cfg5_$TAG.jsonl 2>&1
timeout 600 python bench.py --steps 100 --warmup 10 --cpu-seconds 5 > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
python - <<'PY'
import json, os
tag = os.environ.get("TAG", "perf")
for f in [f"gpurun_out/shapes_{tag}.jsonl", f"gpurun_out/cfg5_{tag}.jsonl"]:
    rows = [json.loads(l) for l in open(f) if l.startswith("{")]
    if "cfg5" in f:
        fr = [r["frac_of_peak"] for r in rows]
        print("cfg5 cells", len(rows), "min frac", round(min(fr), 3) if fr else None, "median", round(sorted(fr)[len(fr)//2], 3) if fr else None)
        for r in sorted(rows, key=lambda r: r["frac_of_peak"])[:12]:
            print("  ", r["case"], round(r["ms_median"], 4), round(r["frac_of_peak"], 3), r["plan"]["kernel"], r["plan"]["group"], r["plan"]["splits"])
    else:
        for r in rows:
            print(r["case"], round(r["ms_median"], 4), round(r["GBps"]), round(r["frac_of_peak"], 3))
b = open(f"gpurun_out/bench_{tag}.json").read().strip()
print(b[:600])
PY
if [ "${NCU:-0}" = "1" ]; then
  mkdir -p gpurun_out/ncu
  timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ncu/launches_$TAG.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu/launches_$TAG.log 2>&1
  for c in "stream_kernel cfg2-f32-sum fp32sum" "col_kernel cfg3-col cfg3col" "stream_kernel cfg3-row cfg3row" "heat cfg4-heat heat" "seg_kernel cfg5-land-int32-v cfg5v"; do
    set -- $c
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:$1 -s 3 -c 1 -o gpurun_out/ncu/$3_$TAG -f python tools/kdriver.py $2 --reps 1 > gpurun_out/ncu/$3_$TAG.log 2>&1
  done
  ls gpurun_out/ncu
fi
