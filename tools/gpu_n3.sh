mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_paper_ab.py tests/test_gpu_multi.py -q -x > gpurun_out/pytest_n3.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_n3.log
tail -3 gpurun_out/pytest_n3.log
timeout 600 python tools/ab_paper.py > gpurun_out/ab_paper_n3.jsonl 2>&1
python - <<'PY'
import json
for l in open("gpurun_out/ab_paper_n3.jsonl"):
    if l.startswith("{"):
        d = json.loads(l); print({k: (round(v, 4) if isinstance(v, float) else v) for k, v in d.items()})
    else:
        print(l.rstrip()[:200])
PY
