#!/bin/bash
# r02aw: rows grid / coltma threshold / stream CTAs-per-SM rule -- parity, smoke, mid-size sweep, cfg5 A/B
O=gpurun_out/r02aw; mkdir -p $O
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "smoke rc=$?" >> $O/smoke.log; tail -n 2 $O/smoke.log
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_packed.py tests/test_gpu_graphs.py tests/test_gpu_round2.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -n 2 $O/pytest.log
timeout 1200 python tools/ab_env.py --cases nest-add-fp32-8192x1x512-v nest-add-fp32-32768x1x128-v nest-add-fp32-4096x1x1024-g nest-add-fp32-16384x1x512-v nest-add-fp32-65536x1x128-v nest-add-fp32-8192x1x1024-g nest-add-fp32-32768x1x512-v nest-add-fp32-131072x1x128-v nest-add-fp32-16384x1x1024-g nest-add-fp32-65536x1x512-v nest-add-fp32-262144x1x128-v \
  --cfg A: --cfg reg:XR_NO_BULK=1,XR_NO_TMA=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_midsize.jsonl
timeout 900 python tools/ab_env.py --cases cfg2-f32-sum cfg3-row cfg5-land-fp32-gwv cfg5-mul-fp64-gwv nest-add-fp32-16777216x1x1-gwv \
  --cfg A: --cfg c2:XR_STREAM_CTAS_PER_SM=2 --rounds 5 --batch 10 2>&1 | tee $O/ab_ctas.jsonl
