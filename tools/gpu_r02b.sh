#!/bin/bash
# r02b: debug the r02a failures (smoke, TMA fallback, fused timeout), per-CTA
# timeline of the stream kernel with / without PDL, bench with PDL, ncu DRAM %
# of the BASELINE configs summarised ON the box (reports are too big to return).
mkdir -p gpurun_out/ncu gpurun_out/prof
TAG=${TAG:-r02b}
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
timeout 600 python -m pytest tests/test_gpu_round2.py tests/test_gpu_graphs.py tests/test_gpu_nccl1.py -q --tb=long > gpurun_out/pytest_new_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_new_$TAG.log
timeout 300 python tools/timeline.py --elements 134217728 268435456 1073741824 --out gpurun_out/timeline_pdl_$TAG.jsonl > /dev/null 2>gpurun_out/timeline_$TAG.err
XR_NO_PDL=1 timeout 300 python tools/timeline.py --elements 134217728 268435456 1073741824 --out gpurun_out/timeline_nopdl_$TAG.jsonl > /dev/null 2>>gpurun_out/timeline_$TAG.err
timeout 300 python tools/fixed_cost.py > gpurun_out/fixed_cost_pdl_$TAG.jsonl 2>&1
XR_NO_PDL=1 timeout 300 python tools/fixed_cost.py > gpurun_out/fixed_cost_nopdl_$TAG.jsonl 2>&1
timeout 600 python bench.py --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_pdl_$TAG.json 2> gpurun_out/bench_$TAG.err
XR_NO_PDL=1 timeout 600 python bench.py --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_nopdl_$TAG.json 2>> gpurun_out/bench_$TAG.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ncu/launches_$TAG.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu/launches_$TAG.log 2>&1
for c in "stream_kernel cfg2-f32-sum" "coltma_kernel cfg3-col" "heat cfg4-heat"; do
  set -- $c
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$1 -s 3 -c 1 -o gpurun_out/ncu/$2_$TAG -f python tools/kdriver.py $2 --reps 1 > gpurun_out/ncu/$2_$TAG.log 2>&1
done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,dram__bytes.sum.per_second,launch__grid_size,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active
for c in cfg2-f32-max cfg2-f32-min cfg2-i64-sum cfg2-i64-max cfg2-i64-min cfg3-row cfg5-mul-int32-g cfg5-and-int32-w cfg5-xor-int32-v cfg5-land-int32-gw cfg5-lor-int32-gv cfg5-mul-fp32-wv cfg5-land-fp32-gwv cfg5-mul-int64-g cfg5-or-int64-w cfg5-xor-int64-v cfg5-mul-fp64-gw cfg5-land-fp64-gv cfg5-lor-fp64-wv cfg5-mul-fp64-gwv; do
  timeout 300 ncu --metrics $M --clock-control none -k regex:"_kernel" -s 3 -c 1 -o gpurun_out/ncu/${c}_$TAG -f python tools/kdriver.py $c --reps 1 > gpurun_out/ncu/${c}_$TAG.log 2>&1
done
python tools/ncu_summary.py $TAG --launches gpurun_out/ncu/launches_$TAG.csv --outdir gpurun_out/prof > gpurun_out/prof/summary_$TAG.log 2>&1
mkdir -p gpurun_out/keep && cp gpurun_out/ncu/cfg2-f32-sum_$TAG.ncu-rep gpurun_out/keep/ 2>/dev/null
rm -f gpurun_out/ncu/*.ncu-rep
du -sh gpurun_out
tail -30 gpurun_out/smoke_$TAG.log; tail -30 gpurun_out/pytest_new_$TAG.log; cat gpurun_out/timeline_pdl_$TAG.jsonl gpurun_out/timeline_nopdl_$TAG.jsonl | cut -c1-600
cat gpurun_out/prof/summary_$TAG.log | head -40
