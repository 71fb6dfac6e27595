#!/bin/bash
O=gpurun_out/r02bh; mkdir -p $O
timeout 1500 python tools/ab_env.py --cases nest-add-fp32-536870x1x250-v nest-add-fp32-268435x1x500-v nest-add-fp32-1073741x1x125-v nest-max-int32-178956x1x750-v nest-add-fp64-268435x1x250-v nest-add-fp32-8192x273x60-gv \
  --cfg A: --cfg w8_1k:XR_SEG_W8_MAX=1024 --cfg w8_4k:XR_SEG_W8_MAX=4096 --rounds 5 --batch 10 2>&1 | tee $O/ab_seg_w8.jsonl
