#!/bin/bash
# r02ai: stream kernel RKR unit order (output-major vs split-major) A/B; split-major coltma default parity
O=gpurun_out/r02ai; mkdir -p $O
timeout 900 python tools/ab_env.py --cases cfg5-land-fp64-gv cfg5-mul-int64-gv cfg5-mul-fp64-gv nest-add-fp32-256x4096x1024-gv \
  --cfg A: --cfg B:XR_STREAM_SPLIT_MAJOR=1 --rounds 7 --batch 10 2>&1 | tee $O/ab_stream_order.jsonl
XR_STREAM_SPLIT_MAJOR=1 XR_SMALL_BYTES=0 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > $O/pytest_smaj.log 2>&1; echo "pytest rc=$?" >> $O/pytest_smaj.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -2 $O/pytest_smaj.log $O/pytest.log
