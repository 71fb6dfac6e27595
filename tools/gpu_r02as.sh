#!/bin/bash
# r02as: column TMA kernel vs the register column kernels, re-checked per shape (interleaved A/B)
O=gpurun_out/r02as; mkdir -p $O
timeout 1500 python tools/ab_env.py --cases cfg5-mul-int32-g cfg5-and-int32-w cfg5-land-int32-gw cfg5-mul-int64-g cfg5-or-int64-w cfg5-mul-fp64-gw cfg3-col \
  nest-add-fp32-256x1x1048576-g nest-max-int32-4096x1x65536-g nest-mul-fp64-64x8192x512-w \
  --cfg A: --cfg noTMA:XR_NO_TMA=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_col.jsonl
