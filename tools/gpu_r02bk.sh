#!/bin/bash
# r02bk: 11 nest shapes x 7 masks (512 MiB fp32 each): absolute rates, to spot slow families
O=gpurun_out/r02bk; mkdir -p $O
timeout 2400 python tools/ab_env.py --cases $(cat tools/cases_r02bk.txt) --cfg A: --rounds 3 --batch 5 2>&1 | tee $O/sweep3.jsonl
