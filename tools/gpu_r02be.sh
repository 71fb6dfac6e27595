#!/bin/bash
# r02be: shape-family sweep 2 (non-power-of-two rows, mid-width columns) vs the register kernels
O=gpurun_out/r02be; mkdir -p $O
timeout 2000 python tools/ab_env.py --cases \
  nest-add-fp32-699050x1x192-g nest-add-fp32-5592405x1x24-g nest-add-fp32-4096x256x128-w nest-add-fp32-536870x1x250-v \
  nest-add-fp32-8192x273x60-gv nest-add-fp64-8192x1x8191-v nest-add-fp32-1x134217727x1-w nest-max-int32-3x44739242x1-gwv \
  nest-add-fp32-16384x8192x1-g nest-xor-int32-1024x1x131071-v \
  --cfg A: --cfg reg:XR_NO_BULK=1,XR_NO_TMA=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_families2.jsonl
