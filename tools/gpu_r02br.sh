#!/bin/bash
O=gpurun_out/r02br; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "shortrow or fuzz or all_pairs" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -n 2 $O/pytest.log
timeout 900 python tools/ab_env.py --cases nest-add-fp32-1024x65536x2-v nest-add-fp32-524288x16x16-v nest-add-fp32-4096x1024x32-v nest-mul-fp64-67108864x1x2-v nest-add-fp64-4194304x1x16-v \
  --cfg A: --rounds 3 --batch 5 2>&1 | tee $O/ab_shortrow2.jsonl
