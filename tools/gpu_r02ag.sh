#!/bin/bash
# r02ag: flat column kernel (contiguous row blocks) vs column TMA kernel on the cfg5 GW / W cells
O=gpurun_out/r02ag; mkdir -p $O
timeout 900 python tools/ab_env.py --cases cfg5-land-int32-gw cfg5-mul-fp32-gw cfg5-mul-int64-gw cfg5-mul-fp64-gw cfg5-and-int32-w cfg5-or-int64-w \
  --cfg A: --cfg B:XR_FLAT_MAX_ROW=4096 --cfg C:XR_FLAT_MAX_ROW=4096,XR_FLAT_UNITS_PER_CTA=2 --rounds 7 --batch 10 2>&1 | tee $O/ab_flat.jsonl
XR_FLAT_MAX_ROW=4096 XR_SMALL_BYTES=0 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -2 $O/pytest.log
