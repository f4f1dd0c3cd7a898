#!/bin/bash
# Fold experiments: per-class rates, skeleton modes, full-size ncu capture of both fold launches.
mkdir -p gpurun_out
for m in 0 1 2; do
  OWL_FOLD_MODE=$m OWL_FOLD_VERBOSE=1 timeout 300 python bench.py --steps 2 --warmup 1 --no-cpu --breakdown > gpurun_out/mode$m.txt 2> gpurun_out/mode$m.err
  python -c "import json;d=json.loads(open('gpurun_out/mode$m.txt').read().strip().splitlines()[-1]);print('mode $m', round(d['ms_per_step'],2), round(d['roofline']['achieved']), d['breakdown_ms'])"
  grep '\[owl\]' gpurun_out/mode$m.err | tail -2
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fold_kernel -c 2 -o gpurun_out/prof_full python bench.py --steps 1 --warmup 0 --no-cpu > gpurun_out/ncu_full2.log 2>&1
tail -1 gpurun_out/ncu_full2.log
