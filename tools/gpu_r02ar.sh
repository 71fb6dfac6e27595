#!/bin/bash
# r02ar: RKR C >= O (2-4 KiB rows) on the seg kernel -- parity + interleaved A/B vs the ring kernels
O=gpurun_out/r02ar; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -n 2 $O/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log; tail -n 2 $O/smoke.log
timeout 900 python tools/ab_env.py --cases cfg5-lor-int32-gv cfg5-mul-fp32-gv cfg5-land-fp64-gv cfg5-mul-int64-gv \
  --cfg A: --cfg ring:XR_RKR_RING=1 --rounds 7 --batch 10 2>&1 | tee $O/ab_rkr_seg.jsonl
