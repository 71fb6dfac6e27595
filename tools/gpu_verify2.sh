#!/bin/bash
# Round-2 verification at HEAD: smoke, full GPU suite, bench (N=1, comm path,
# reference arm), cfg1 graph latency, shape + cfg5 timings, ncu launch list and
# DRAM % of every BASELINE config's kernel (summarised on the box: the reports
# are too large to bring back).
mkdir -p gpurun_out/ncu gpurun_out/prof
TAG=${TAG:-r02v}
KRE='regex:stream_kernel|seg_kernel|coltma_kernel|col_kernel|colflat_kernel|colsmall_kernel|rows_kernel|rkr_kernel|heat_'
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?" >> gpurun_out/bench_$TAG.err
timeout 600 python bench.py --force-comm --steps 100 --no-cpu-baseline > gpurun_out/bench_comm_$TAG.json 2> gpurun_out/bench_comm_$TAG.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$TAG.json 2> gpurun_out/bench_ref_$TAG.err
timeout 300 python tools/bench_graph.py > gpurun_out/graph_$TAG.jsonl 2>&1
timeout 600 python tools/kdriver.py cfg2-f32-sum cfg2-f32-max cfg2-f32-min cfg2-i64-sum cfg2-i64-max cfg2-i64-min cfg2-f64-sum cfg3-row cfg3-col cfg4-heat cfg1-g cfg1-w cfg1-v cfg1-gwv --reps 20 --time > gpurun_out/shapes_$TAG.jsonl 2>&1
timeout 900 python tools/kdriver.py cfg5-all --reps 9 --time > gpurun_out/cfg5_$TAG.jsonl 2>&1
timeout 600 python tools/fixed_cost.py > gpurun_out/fixed_cost_$TAG.jsonl 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ncu/launches_$TAG.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu/launches_$TAG.log 2>&1
for c in cfg2-f32-sum cfg3-col cfg4-heat; do
  timeout 600 ncu --set full --clock-control none --import-source on -k "$KRE" -s 3 -c 1 -o gpurun_out/ncu/${c}_$TAG -f python tools/kdriver.py $c --reps 1 > gpurun_out/ncu/${c}_$TAG.log 2>&1
done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,dram__bytes.sum.per_second,launch__grid_size,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active
for c in cfg2-f32-max cfg2-f32-min cfg2-i64-sum cfg2-i64-max cfg2-i64-min cfg2-f64-sum cfg3-row \
         cfg5-mul-int32-g cfg5-and-int32-w cfg5-xor-int32-v cfg5-land-int32-gw cfg5-lor-int32-gv cfg5-mul-fp32-wv cfg5-land-fp32-gwv \
         cfg5-mul-int64-g cfg5-or-int64-w cfg5-xor-int64-v cfg5-mul-fp64-gw cfg5-land-fp64-gv cfg5-lor-fp64-wv cfg5-mul-fp64-gwv; do
  timeout 300 ncu --metrics $M --clock-control none -k "$KRE" -s 3 -c 1 -o gpurun_out/ncu/${c}_$TAG -f python tools/kdriver.py $c --reps 1 > gpurun_out/ncu/${c}_$TAG.log 2>&1
done
python tools/ncu_summary.py $TAG --launches gpurun_out/ncu/launches_$TAG.csv --outdir gpurun_out/prof > gpurun_out/prof/summary_$TAG.log 2>&1
mkdir -p gpurun_out/keep && cp gpurun_out/ncu/cfg2-f32-sum_$TAG.ncu-rep gpurun_out/keep/ 2>/dev/null
rm -f gpurun_out/ncu/*.ncu-rep
du -sh gpurun_out
tail -2 gpurun_out/smoke_$TAG.log; tail -14 gpurun_out/pytest_gpu_$TAG.log
cut -c1-300 gpurun_out/bench_$TAG.json; cut -c1-300 gpurun_out/bench_ref_$TAG.json
grep "DRAM %" -A 30 gpurun_out/prof/ncu_$TAG.md | cut -c1-140
