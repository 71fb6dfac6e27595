#!/bin/bash
# r02ba: narrow-row rkr consumers -- parity + A/B vs the seg kernel on large narrow RKR shapes
O=gpurun_out/r02ba; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "rkr" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -n 3 $O/pytest.log
timeout 1200 python tools/ab_env.py --cases nest-add-fp32-8192x256x64-gv nest-add-fp32-64x65536x32-gv nest-max-int32-128x65536x16-gv nest-mul-fp64-4096x1024x16-gv nest-xor-int64-512x16384x8-gv nest-add-fp32-2048x2048x32-gv \
  --cfg A: --cfg seg:XR_NO_RKR_NARROW=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_narrow.jsonl
