#!/bin/bash
# r02aj: split-major column kernel -- units per CTA re-sweep (interleaved A/B)
O=gpurun_out/r02aj; mkdir -p $O
timeout 900 python tools/ab_env.py --cases cfg5-land-int32-gw cfg5-mul-fp64-gw cfg3-col \
  --cfg A: --cfg k4:XR_COLTMA_UNITS_PER_CTA=4 --cfg k8:XR_COLTMA_UNITS_PER_CTA=8 --cfg k16:XR_COLTMA_UNITS_PER_CTA=16 --cfg k32:XR_COLTMA_UNITS_PER_CTA=32 --rounds 5 --batch 10 2>&1 | tee $O/ab_k.jsonl
