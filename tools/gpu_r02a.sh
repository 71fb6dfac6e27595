#!/bin/bash
# r02a: first GPU pass of round 2 -- smoke, the new round-2 tests, the full GPU
# suite, bench (N=1, and the comm path at 1 rank), ncu DRAM % per BASELINE config.
mkdir -p gpurun_out/ncu
TAG=${TAG:-r02a}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu_$TAG.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_$TAG.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke_$TAG.log
timeout 900 python -m pytest tests/test_gpu_round2.py tests/test_gpu_nccl1.py tests/test_gpu_fused.py -q -x > gpurun_out/pytest_new_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_new_$TAG.log
timeout 2400 python -m pytest tests -m gpu -q --durations=10 > gpurun_out/pytest_gpu_$TAG.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_$TAG.log
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err; echo "bench rc=$?" >> gpurun_out/bench_$TAG.err
timeout 600 python bench.py --force-comm --steps 50 --no-cpu-baseline > gpurun_out/bench_comm_$TAG.json 2> gpurun_out/bench_comm_$TAG.err; echo "rc=$?" >> gpurun_out/bench_comm_$TAG.err
timeout 300 python bench.py --gpus 2 > gpurun_out/bench_g2_$TAG.json 2> gpurun_out/bench_g2_$TAG.err; echo "rc=$?" >> gpurun_out/bench_g2_$TAG.err
# ncu: launch list of the bench command + DRAM % of every BASELINE config's kernel
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ncu/launches_$TAG.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 0 > gpurun_out/ncu/launches_$TAG.log 2>&1
for c in "stream_kernel cfg2-f32-sum" "coltma_kernel cfg3-col" "heat cfg4-heat"; do
  set -- $c
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:$1 -s 3 -c 1 -o gpurun_out/ncu/$2_$TAG -f python tools/kdriver.py $2 --reps 1 > gpurun_out/ncu/$2_$TAG.log 2>&1
done
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,dram__bytes.sum.per_second,launch__grid_size,launch__registers_per_thread,sm__warps_active.avg.pct_of_peak_sustained_active
for c in cfg2-f32-max cfg2-f32-min cfg2-i64-sum cfg2-i64-max cfg3-row cfg5-mul-int32-g cfg5-and-int32-w cfg5-xor-int32-v cfg5-land-int32-gw cfg5-lor-int32-gv cfg5-mul-fp32-wv cfg5-land-fp32-gwv cfg5-mul-int64-g cfg5-or-int64-w cfg5-xor-int64-v cfg5-mul-fp64-gw cfg5-land-fp64-gv cfg5-lor-fp64-wv cfg5-mul-fp64-gwv; do
  timeout 300 ncu --metrics $M --clock-control none -k regex:"kernel" -s 3 -c 1 -o gpurun_out/ncu/${c}_$TAG -f python tools/kdriver.py $c --reps 1 > gpurun_out/ncu/${c}_$TAG.log 2>&1
done
cat gpurun_out/smoke_$TAG.log | tail -3; tail -5 gpurun_out/pytest_new_$TAG.log; tail -14 gpurun_out/pytest_gpu_$TAG.log
cat gpurun_out/bench_$TAG.json gpurun_out/bench_comm_$TAG.json; tail -3 gpurun_out/bench_g2_$TAG.err; ls gpurun_out/ncu | wc -l
