mkdir -p gpurun_out
timeout 900 python tools/kdriver.py cfg5-all --reps 15 --time > gpurun_out/cfg5_r01zc.jsonl 2>&1
timeout 900 python tools/kdriver.py cfg2-f32-sum cfg3-row cfg3-col cfg4-heat --reps 20 --time > gpurun_out/shapes_r01zc.jsonl 2>&1
tail -2 gpurun_out/cfg5_r01zc.jsonl
