#!/bin/bash
O=gpurun_out/r02at; mkdir -p $O
timeout 900 python tools/ab_env.py --cases nest-max-int32-4096x1x65536-g nest-mul-fp64-64x8192x512-w nest-add-fp32-2048x1x131072-g \
  --cfg A: --cfg g444:XR_COLTMA_GRID=444 --cfg k4:XR_COLTMA_UNITS_PER_CTA=4 --cfg k8:XR_COLTMA_UNITS_PER_CTA=8 --rounds 5 --batch 10 2>&1 | tee $O/ab_grid.jsonl
