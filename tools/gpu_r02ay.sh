#!/bin/bash
# r02ay: wide-row column plans (RK with 2 / 4 KiB rows as contiguous 1 KiB box rows)
O=gpurun_out/r02ay; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "coltma_box_order_group or all_pairs or fuzz" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -n 2 $O/pytest.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -x -k "cfg5" > $O/pytest_full.log 2>&1; echo "pytest rc=$?" >> $O/pytest_full.log
tail -n 2 $O/pytest_full.log
timeout 900 python tools/ab_env.py --cases cfg5-land-int32-gw cfg5-mul-fp32-gw cfg5-mul-fp64-gw cfg5-mul-int64-gw \
  --cfg A: --cfg nowide:XR_COLTMA_NO_WIDE=1 --cfg k4:XR_COLTMA_UNITS_PER_CTA=4 --cfg k8:XR_COLTMA_UNITS_PER_CTA=8 --rounds 5 --batch 10 2>&1 | tee $O/ab_wide.jsonl
timeout 900 python tools/ab_env.py --single --cases cfg5-land-int32-gw cfg5-mul-fp64-gw \
  --cfg A: --cfg nowide:XR_COLTMA_NO_WIDE=1 --rounds 5 --batch 7 2>&1 | tee $O/ab_wide_single.jsonl
