#!/bin/bash
# odd-width heat (4-CTA bounds on the odd instantiation) timings, then the full GPU suite at the final tree
TAG=r01zg bash tools/gpu_heat_odd.sh
timeout 2400 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu_r01zg.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_r01zg.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" >> gpurun_out/pytest_gpu_r01zg.log 2>&1
tail -4 gpurun_out/pytest_gpu_r01zg.log
