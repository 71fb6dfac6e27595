#!/bin/bash
# r02c: PDL on every kernel + guided units for the whole-array stream -- the
# GPU suite, smoke, per-CTA timeline, fixed cost, bench, cfg5 / shape timings.
mkdir -p gpurun_out
TAG=${TAG:-r02c}
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
timeout 2400 python -m pytest tests -m gpu -q -x --durations=10 > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 300 python tools/timeline.py --elements 134217728 268435456 1073741824 --out gpurun_out/timeline_$TAG.jsonl > /dev/null 2>gpurun_out/timeline_$TAG.err
timeout 300 python tools/fixed_cost.py > gpurun_out/fixed_cost_$TAG.jsonl 2>&1
XR_NO_GUIDED=1 timeout 300 python tools/fixed_cost.py > gpurun_out/fixed_cost_noguided_$TAG.jsonl 2>&1
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
timeout 600 python tools/kdriver.py cfg2-f32-sum cfg2-f32-max cfg2-f32-min cfg2-i64-sum cfg2-i64-max cfg2-i64-min cfg2-f64-sum cfg3-row cfg3-col cfg4-heat cfg1-g cfg1-w cfg1-v cfg1-gwv --reps 20 --time > gpurun_out/shapes_$TAG.jsonl 2>&1
timeout 900 python tools/kdriver.py cfg5-all --reps 9 --time > gpurun_out/cfg5_$TAG.jsonl 2>&1
tail -3 gpurun_out/smoke_$TAG.log; tail -16 gpurun_out/pytest_gpu_$TAG.log; cut -c1-700 gpurun_out/timeline_$TAG.jsonl
cat gpurun_out/fixed_cost_$TAG.jsonl gpurun_out/fixed_cost_noguided_$TAG.jsonl | cut -c1-300; cut -c1-400 gpurun_out/bench_$TAG.json
