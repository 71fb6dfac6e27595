#!/bin/bash
# r02ao: rkr kernel (32-bit GV) units per CTA x grid, interleaved A/B
O=gpurun_out/r02ao; mkdir -p $O
timeout 900 python tools/ab_env.py --cases cfg5-lor-int32-gv cfg5-mul-fp32-gv \
  --cfg A: --cfg k2:XR_RKR_UNITS_PER_CTA=2 --cfg k3:XR_RKR_UNITS_PER_CTA=3 --cfg k6:XR_RKR_UNITS_PER_CTA=6 --cfg k8:XR_RKR_UNITS_PER_CTA=8 \
  --cfg g444:XR_RKR_GRID=444 --cfg g148:XR_RKR_GRID=148 --cfg stream:XR_NO_RKR=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_rkr.jsonl
