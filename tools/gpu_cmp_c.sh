mkdir -p gpurun_out/ncu
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "stream_rkr or rows_kernel or all_pairs or fuzz or ring" > gpurun_out/pytest_c.log 2>&1; tail -2 gpurun_out/pytest_c.log
for c in cfg5-add-int32-v cfg5-land-fp32-v cfg5-mul-int64-gv cfg5-land-fp64-gv cfg5-lor-fp64-v cfg5-lor-int64-v cfg5-add-fp64-v; do timeout 120 python tools/kdriver.py $c --reps 15 --time; done > gpurun_out/cells_c.jsonl 2>&1
python -c "
import json
for l in open('gpurun_out/cells_c.jsonl'):
    if l.startswith('{'):
        d=json.loads(l); print(d['case'], round(d['ms_median']*1e3,1), round(d['frac_of_peak'],3), d['plan']['kernel'], d['plan']['splits'], d['plan']['units'])
"
for t in new old; do D=.; [ $t = old ] && D=abold
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:seg_kernel -s 3 -c 1 -o gpurun_out/ncu/lorf64v_$t -f python $D/tools/kdriver.py cfg5-lor-fp64-v --reps 1 > gpurun_out/ncu/lorf64v_$t.log 2>&1
  timeout 300 ncu --set full --clock-control none --import-source on -k regex:seg_kernel -s 3 -c 1 -o gpurun_out/ncu/lori64v_$t -f python $D/tools/kdriver.py cfg5-lor-int64-v --reps 1 > gpurun_out/ncu/lori64v_$t.log 2>&1
done
ls gpurun_out/ncu
