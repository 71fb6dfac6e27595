#!/bin/bash
# r02z: sharded unit scheduler -- parity of the ring kernels, unit-size sweeps
O=gpurun_out/r02z; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py tests/test_gpu_graphs.py tests/test_gpu_round2.py -q -x > $O/pytest.log 2>&1; echo "pytest rc=$?" >> $O/pytest.log
tail -3 $O/pytest.log
sw() {  # env-spec case...
  local spec=$1; shift
  for c in "$@"; do
    env $spec timeout 300 python tools/kdriver.py $c --reps 15 --time 2>&1 | python -c "
import sys,json
for l in sys.stdin:
    try: d=json.loads(l)
    except Exception: continue
    print('$spec', d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3))"
  done
}
for sp in 4096 8192 16384 32768 65536; do
  sw XR_STREAM_SPLITS=$sp nest-add-fp32-134217728x1x1-gwv nest-xor-int32-134217728x1x1-gwv nest-add-fp32-268435456x1x1-gwv nest-mul-fp64-134217728x1x1-gwv
done | tee $O/stream_splits.txt
for k in 2 4 8 16 32 64; do
  sw XR_COLTMA_UNITS_PER_CTA=$k cfg5-mul-int64-g cfg5-mul-fp64-gw cfg5-mul-int32-g cfg5-land-int32-gw
done | tee $O/coltma_units.txt
for k in 4 8 16 32; do
  sw XR_RKR_UNITS_PER_CTA=$k cfg5-lor-int32-gv cfg5-mul-fp32-gv
done | tee $O/rkr_units.txt
