#!/bin/bash
# r02bg: flat column kernel for non-power-of-two rows -- parity + A/B vs the register column kernel
O=gpurun_out/r02bg; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_packed.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -n 2 $O/pytest.log
timeout 1200 python tools/ab_env.py --cases nest-add-fp32-5592405x1x24-g nest-add-fp32-699050x1x192-g nest-max-int32-2796202x1x48-g nest-mul-fp64-1398101x1x48-g nest-add-fp32-1747626x1x80-g nest-add-int32-1048576x2x32-g \
  --cfg A: --cfg old:XR_NO_FLAT_NPOW2=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_flat_npow2.jsonl
