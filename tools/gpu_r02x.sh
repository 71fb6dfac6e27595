#!/bin/bash
# r02x: packed int32 '+' gang tier (parity + cfg1 graph latency), coltma / stream
# per-CTA timelines of the 1 GiB cfg5 cells.
mkdir -p gpurun_out/r02x
O=gpurun_out/r02x
timeout 900 python -m pytest tests/test_gpu_packed.py tests/test_gpu_graphs.py tests/test_gpu_parity.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
timeout 300 python tools/bench_graph.py > $O/graph.jsonl 2>&1
XR_NO_PACKED=1 timeout 300 python tools/bench_graph.py > $O/graph_nopacked.jsonl 2>&1
cat $O/graph.jsonl; echo ---; cat $O/graph_nopacked.jsonl
for m in g w gw gv wv gwv v; do
  timeout 300 python tools/timeline.py --nest 512 512 512 --mask $m --dtype fp64 --reps 10 >> $O/timeline_fp64.jsonl 2>&1
done
for m in g w gw gv gwv; do
  timeout 300 python tools/timeline.py --nest 512 512 512 --mask $m --dtype fp32 --reps 10 >> $O/timeline_fp32.jsonl 2>&1
done
python - <<'PY'
import json
for f in ("gpurun_out/r02x/timeline_fp64.jsonl", "gpurun_out/r02x/timeline_fp32.jsonl"):
    for l in open(f):
        try: d = json.loads(l)
        except Exception: print(l.strip()[:200]); continue
        print(d["dtype"], d["mask"], d["plan"], "ev", round(d["event_ms_median"]*1e3,1), "span", d["span_us_first_start_to_out"],
              "start", d["cta_start_us"].get("p100"), "cons_end", d["cons_end_us"], "claim_last", d.get("last_real_claim_us"),
              "upc", d["units_per_cta"], "unit_us", d["unit_us"])
PY
# heat: odd (8191^2) vs even (8192^2) full captures, details pages only
for c in heat-8191 cfg4-heat; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat_ -s 3 -c 1 -o $O/$c -f python tools/kdriver.py $c --reps 1 > $O/ncu_$c.log 2>&1
  ncu -i $O/$c.ncu-rep --page details --csv > $O/${c}_details.csv 2>&1
  ncu -i $O/$c.ncu-rep --page source --csv --print-source sass > $O/${c}_sass.csv 2>&1
  rm -f $O/$c.ncu-rep
done
du -sh $O
# per-unit cost of the stream kernel: equal units of 128 / 64 / 32 / 16 KiB at 512 MiB and 1 GiB
for sp in 4096 8192 16384 32768 65536; do
  for c in nest-add-fp32-134217728x1x1-gwv nest-xor-int32-134217728x1x1-gwv nest-add-fp32-268435456x1x1-gwv; do
    XR_STREAM_SPLITS=$sp timeout 300 python tools/kdriver.py $c --reps 15 --time 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print('splits $sp', d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3))"
  done
done | tee $O/stream_splits.txt
