#!/bin/bash
# GPU pass 2: all GPU tests (incl. full sizes), per-shape timings, ncu launch list + full captures
mkdir -p gpurun_out/ncu
timeout 2400 python -m pytest tests -m gpu -q --durations=20 > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
tail -25 gpurun_out/pytest_gpu.log
timeout 600 python tools/kdriver.py cfg2-f32-sum cfg2-f32-max cfg2-f32-min cfg2-i64-sum cfg2-i64-max cfg2-i64-min cfg3-row cfg3-col cfg4-heat cfg1-g cfg1-w cfg1-v cfg1-gwv --reps 20 --time > gpurun_out/shapes.jsonl 2>&1
timeout 900 python tools/kdriver.py cfg5-all --reps 7 --time > gpurun_out/cfg5.jsonl 2>&1
# launch list of the bench command (cold-cache, serialised)
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ncu/launches_r01.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu/launches_bench.log 2>&1
# one full capture per dominant kernel
timeout 600 ncu --set full --clock-control none --import-source on -k regex:seg_kernel -s 3 -c 1 -o gpurun_out/ncu/fp32sum_r01 -f python tools/kdriver.py cfg2-f32-sum --reps 1 > gpurun_out/ncu/fp32sum.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:col_kernel -s 3 -c 1 -o gpurun_out/ncu/cfg3col_r01 -f python tools/kdriver.py cfg3-col --reps 1 > gpurun_out/ncu/cfg3col.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:seg_kernel -s 3 -c 1 -o gpurun_out/ncu/cfg3row_r01 -f python tools/kdriver.py cfg3-row --reps 1 > gpurun_out/ncu/cfg3row.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:heat_kernel -s 3 -c 1 -o gpurun_out/ncu/heat_r01 -f python tools/kdriver.py cfg4-heat --reps 1 > gpurun_out/ncu/heat.log 2>&1
cat gpurun_out/shapes.jsonl | python -c "import sys,json; [print(d['case'], round(d['ms_median'],4), round(d['GBps']), round(d['frac_of_peak'],3)) for d in map(json.loads, sys.stdin) if d]"
ls -la gpurun_out/ncu
