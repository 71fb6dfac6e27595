#!/bin/bash
# r02aq: RKR shapes (gang + vector reduced) -- ring kernels (rkr / stream) vs the register seg kernel
O=gpurun_out/r02aq; mkdir -p $O
timeout 1700 python tools/ab_env.py --cases \
  nest-lor-int32-512x256x512-gv nest-lor-int32-512x512x512-gv nest-lor-int32-1024x512x512-gv nest-lor-int32-256x1024x512-gv nest-lor-int32-128x2048x512-gv nest-lor-int32-2048x256x512-gv \
  nest-mul-fp64-512x128x512-gv nest-mul-fp64-512x256x512-gv nest-mul-fp64-512x512x512-gv nest-mul-fp64-256x1024x512-gv nest-mul-fp64-128x2048x512-gv nest-mul-fp64-1024x512x512-gv \
  --cfg A: --cfg seg:XR_NO_BULK=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_rkr_shapes.jsonl
