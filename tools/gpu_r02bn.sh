#!/bin/bash
O=gpurun_out/r02bn; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "thincol or all_pairs or fuzz or cfg1 or coltma" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -n 2 $O/pytest.log
timeout 900 python tools/ab_env.py --cases nest-add-fp32-2x65536x1024-g nest-add-fp32-524288x16x16-w nest-max-int32-8x1x16777216-g nest-mul-fp64-32x1x2097152-g nest-add-fp32-16x4096x2048-w \
  --cfg A: --cfg old:XR_NO_THINCOL=1 --rounds 5 --batch 5 2>&1 | tee $O/ab_thincol.jsonl
