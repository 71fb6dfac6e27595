#!/bin/bash
O=gpurun_out/r02au; mkdir -p $O
timeout 900 python tools/ab_env.py --cases cfg2-f32-sum cfg5-land-fp32-gwv cfg5-mul-fp64-gwv cfg5-lor-fp64-wv cfg5-mul-fp32-wv \
  --cfg A: --cfg c3:XR_STREAM_CTAS_PER_SM=3 --rounds 5 --batch 10 2>&1 | tee $O/ab_stream_ctas.jsonl
timeout 900 python tools/ab_env.py --cases cfg5-xor-int32-v cfg5-mul-fp32-v nest-add-fp32-8192x1x512-v \
  --cfg A: --cfg u16:XR_ROWS_UNITS_PER_CTA=16 --cfg u64:XR_ROWS_UNITS_PER_CTA=64 --cfg seg:XR_NO_BULK=1 --rounds 5 --batch 10 2>&1 | tee $O/ab_rows.jsonl
