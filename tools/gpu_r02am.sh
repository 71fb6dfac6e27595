#!/bin/bash
# r02am: per-plan column group size (16 when S > 64) -- parity + interleaved A/B
O=gpurun_out/r02am; mkdir -p $O
XR_SMALL_BYTES=0 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > $O/pytest_staged.log 2>&1; echo "pytest rc=$?" >> $O/pytest_staged.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "cfg5 or cfg3" > $O/pytest_full.log 2>&1; echo "pytest rc=$?" >> $O/pytest_full.log
tail -n 2 $O/pytest_staged.log; tail -n 2 $O/pytest_full.log
timeout 900 python tools/ab_env.py --cases cfg5-land-int32-gw cfg5-mul-fp32-gw cfg5-or-int32-gw cfg5-mul-fp64-gw cfg3-col \
  --cfg A: --cfg g64:XR_COLTMA_GROUP=64 --rounds 7 --batch 10 2>&1 | tee $O/ab_group.jsonl
