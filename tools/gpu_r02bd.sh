#!/bin/bash
O=gpurun_out/r02bd; mkdir -p $O
timeout 1500 python tools/ab_env.py --cases nest-add-fp32-65536x1x2048-v nest-add-fp64-65536x1x1024-v nest-add-fp32-16384x1x4096-v nest-add-fp32-32768x1x4096-v nest-max-int32-8192x1x8192-v nest-add-fp32-4096x1x8192-v \
  --cfg A: --cfg w16k:XR_SEG_W32_MAX=16384 --cfg w64k:XR_SEG_W32_MAX=65536 --rounds 5 --batch 10 2>&1 | tee $O/ab_seg_w.jsonl
