#!/bin/bash
# r02ax: column-kernel r02 choices in SINGLE-launch timing (as ncu and the cfg5 tables see them)
O=gpurun_out/r02ax; mkdir -p $O
timeout 1500 python tools/ab_env.py --single --cases cfg5-land-int32-gw cfg5-mul-fp32-gw cfg5-mul-fp64-gw cfg5-mul-int32-g cfg5-and-int32-w cfg5-or-int64-w cfg3-col \
  --cfg A: --cfg tile:XR_COLTMA_TILE_MAJOR=1 --cfg g64:XR_COLTMA_GROUP=64 --cfg old:XR_COLTMA_TILE_MAJOR=1,XR_COLTMA_GROUP=64 --rounds 5 --batch 7 2>&1 | tee $O/ab_single_col.jsonl
timeout 900 python tools/ab_env.py --single --cases cfg5-land-fp32-gwv cfg5-mul-fp64-gwv cfg5-lor-int32-gv cfg5-land-fp64-gv \
  --cfg A: --cfg c2:XR_STREAM_CTAS_PER_SM=2 --cfg ring:XR_RKR_RING=1 --rounds 5 --batch 7 2>&1 | tee $O/ab_single_stream.jsonl
