#!/bin/bash
O=gpurun_out/r02bc; mkdir -p $O
XR_SEG_STATIC=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "all_pairs or fuzz or init_from_out" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -n 2 $O/pytest.log
timeout 1200 python tools/ab_env.py --cases nest-add-fp32-16384x1x4096-v nest-add-fp32-8192x1x8192-v nest-add-fp64-65536x1x1024-v nest-max-int32-131072x1x1024-v nest-add-fp32-2048x1x16384-v nest-add-fp32-65536x1x2048-v \
  --cfg A: --cfg static:XR_SEG_STATIC=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_seg_static.jsonl
