#!/bin/bash
# r02az: broad shape-family sweep -- planner's choice vs the register kernels (XR_NO_BULK + XR_NO_TMA)
O=gpurun_out/r02az; mkdir -p $O
timeout 2000 python tools/ab_env.py --cases \
  nest-add-fp32-1048576x1x64-g nest-add-fp32-4194304x1x16-g nest-max-int32-67108864x1x4-g nest-add-fp64-512x1024x64-w \
  nest-add-fp32-16384x1x4096-v nest-add-fp32-4096x1x16384-v nest-add-fp32-256x1x262144-v nest-add-fp32-64x1x1048576-v nest-add-fp32-8x1x16777216-v \
  nest-add-fp32-8192x256x64-gv nest-add-fp32-64x65536x32-gv nest-add-fp32-1024x1024x64-gw nest-add-fp32-64x1024x2048-wv \
  nest-add-fp64-64x2048x1024-gv nest-add-fp64-2048x64x1024-gv nest-xor-int64-16x1024x8192-gv \
  --cfg A: --cfg reg:XR_NO_BULK=1,XR_NO_TMA=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_families.jsonl
