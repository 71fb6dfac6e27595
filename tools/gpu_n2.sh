mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_multi.py tests/test_gpu_n1.py tests/test_gpu_parity.py -q -x -m "gpu and not slow" > gpurun_out/pytest_n2.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_n2.log
tail -3 gpurun_out/pytest_n2.log
timeout 300 python tools/bench_multi.py > gpurun_out/multi_n2.jsonl 2>&1
cat gpurun_out/multi_n2.jsonl | cut -c1-300
