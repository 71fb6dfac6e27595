#!/bin/bash
# r02bj: narrow rkr consumers for non-power-of-two rows -- parity + A/B vs the seg kernel
O=gpurun_out/r02bj; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py -q -x -k "rkr" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -n 2 $O/pytest.log
timeout 1200 python tools/ab_env.py --cases nest-add-fp32-8192x273x60-gv nest-add-int64-500x1000x30-gv nest-add-fp32-300x700x100-gv nest-add-fp32-64x65536x32-gv nest-add-fp32-8192x256x64-gv \
  --cfg A: --cfg seg:XR_NO_RKR_NARROW=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_narrow_npow2.jsonl
