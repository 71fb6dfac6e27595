#!/bin/bash
O=gpurun_out/r02bm; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "shortrow or rkr or all_pairs or fuzz or init_from_out or cfg1" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -n 2 $O/pytest.log
timeout 900 python tools/ab_env.py --cases nest-max-fp64-4096x1024x16-gv nest-min-fp64-2048x1024x30-gv nest-max-fp32-8192x256x64-gv \
  --cfg A: --cfg seg:XR_NO_RKR_NARROW=1 --rounds 5 --batch 5 2>&1 | tee $O/ab_rkr_narrow_maxmin.jsonl
