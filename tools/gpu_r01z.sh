#!/bin/bash
# ring kernels (epilogue warp, batched smem loads): parity (full GPU suite) + cfg5 / shape timings
mkdir -p gpurun_out
timeout 900 python tools/kdriver.py cfg5-all --reps 15 --time > gpurun_out/cfg5.jsonl 2>&1
timeout 600 python tools/kdriver.py cfg2-f32-sum cfg2-f32-max cfg2-f32-min cfg2-i64-sum cfg2-i64-max cfg2-i64-min cfg3-row cfg3-col cfg4-heat cfg1-g cfg1-w cfg1-v cfg1-gwv --reps 20 --time > gpurun_out/shapes.jsonl 2>&1
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -5 gpurun_out/pytest_gpu.log
python - <<'PY'
import json, statistics
rows=[json.loads(l) for l in open('gpurun_out/cfg5.jsonl') if l.startswith('{')]
print('cfg5 n', len(rows), 'median', round(statistics.median(r['frac_of_peak'] for r in rows),3), 'min', round(min(r['frac_of_peak'] for r in rows),3))
for r in sorted(rows, key=lambda r: r['frac_of_peak'])[:40]:
    print(r['case'], round(r['ms_median']*1e3,1), round(r['frac_of_peak'],3), r['plan']['kernel'], r['plan']['splits'], r['plan']['units'])
for l in open('gpurun_out/shapes.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print(d['case'], round(d['ms_median']*1e3,1), 'us', round(d['frac_of_peak'],3))
PY
