#!/bin/bash
O=gpurun_out/r02bb; mkdir -p $O
timeout 1200 python tools/ab_env.py --cases nest-add-fp32-8192x256x64-gv nest-add-fp32-64x65536x32-gv nest-mul-fp64-4096x1024x16-gv nest-xor-int64-512x16384x8-gv \
  --cfg A: --cfg k2:XR_RKR_UNITS_PER_CTA=2 --cfg k8:XR_RKR_UNITS_PER_CTA=8 --cfg g444:XR_RKR_GRID=444 --cfg g444k8:XR_RKR_GRID=444,XR_RKR_UNITS_PER_CTA=8 --rounds 5 --batch 10 2>&1 | tee $O/ab_narrow_tune.jsonl
