#!/bin/bash
# Round-end verification at HEAD: smoke, full GPU suite, default bench, reference arm,
# launch list + ncu --set full captures of the top kernels, cfg5/shape timings.
mkdir -p gpurun_out/ncu
TAG=${TAG:-final}
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?" >> gpurun_out/bench_$TAG.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$TAG.json 2> gpurun_out/bench_ref_$TAG.err
timeout 600 python tools/kdriver.py cfg2-f32-sum cfg2-f32-max cfg2-f32-min cfg2-i64-sum cfg2-i64-max cfg2-i64-min cfg2-f64-sum cfg3-row cfg3-col cfg4-heat cfg1-g cfg1-w cfg1-v cfg1-gwv --reps 20 --time > gpurun_out/shapes_$TAG.jsonl 2>&1
timeout 900 python tools/kdriver.py cfg5-all --reps 9 --time > gpurun_out/cfg5_$TAG.jsonl 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ncu/launches_$TAG.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu/launches_$TAG.log 2>&1
for c in "stream_kernel cfg2-f32-sum fp32sum" "col_kernel cfg3-col cfg3col" "heat cfg4-heat heat"; do
  set -- $c
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$1 -s 3 -c 1 -o gpurun_out/ncu/$3_$TAG -f python tools/kdriver.py $2 --reps 1 > gpurun_out/ncu/$3_$TAG.log 2>&1
done
tail -3 gpurun_out/smoke_$TAG.log; tail -14 gpurun_out/pytest_gpu_$TAG.log; cat gpurun_out/bench_$TAG.json gpurun_out/bench_ref_$TAG.json; ls gpurun_out/ncu
