#!/bin/bash
O=gpurun_out/r02bp; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_packed.py -q -x -k "colflat or all_pairs or fuzz or cfg1 or init_from_out or packed" > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -n 2 $O/pytest.log
timeout 900 python tools/ab_env.py --cases nest-add-fp32-1024x65536x2-gw nest-add-fp32-1024x65536x2-w nest-max-int32-1x67108863x2-w \
  --cfg A: --cfg old:XR_NO_FLAT8=1 --rounds 5 --batch 5 2>&1 | tee $O/ab_flat8.jsonl
