#!/bin/bash
# r02ah: column TMA kernel unit order (tile-major vs split-major) -- interleaved A/B + parity
O=gpurun_out/r02ah; mkdir -p $O
timeout 900 python tools/ab_env.py --cases cfg3-col cfg5-land-int32-gw cfg5-mul-fp32-gw cfg5-mul-fp64-gw cfg5-mul-int64-gw cfg5-mul-int32-g \
  --cfg A: --cfg B:XR_COLTMA_SPLIT_MAJOR=1 --rounds 7 --batch 10 2>&1 | tee $O/ab_order.jsonl
XR_COLTMA_SPLIT_MAJOR=1 XR_SMALL_BYTES=0 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -2 $O/pytest.log
