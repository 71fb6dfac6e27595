#!/bin/bash
# r02ap: ring kernels vs register kernels, re-checked per cfg5 shape (interleaved A/B)
O=gpurun_out/r02ap; mkdir -p $O
timeout 1500 python tools/ab_env.py --cases cfg5-lor-int32-gv cfg5-mul-fp32-gv nest-xor-int32-512x512x256-gv nest-add-fp32-1024x1024x128-gv nest-max-fp32-256x4096x512-gv \
  cfg5-land-fp64-gv cfg5-mul-fp32-wv cfg5-lor-fp64-wv cfg5-land-fp32-gwv cfg5-mul-fp64-gwv cfg5-xor-int32-v cfg5-xor-int64-v cfg2-f32-sum \
  --cfg A: --cfg noRKR:XR_NO_RKR=1 --cfg noBULK:XR_NO_BULK=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_ring_vs_reg.jsonl
