#!/bin/bash
# Iteration check: GPU parity tests, bench modes (0 full, 1 no address inserts, 2 stream only), ncu of both folds.
mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -q -x --timeout 60 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
tail -3 gpurun_out/pytest_gpu.txt
for m in 0 1 2; do
  OWL_FOLD_MODE=$m OWL_FOLD_VERBOSE=1 timeout 150 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e --breakdown > gpurun_out/mode$m.txt 2> gpurun_out/mode$m.err
  python -c "import json;d=json.loads(open('gpurun_out/mode$m.txt').read().strip().splitlines()[-1]);print('mode $m', round(d['ms_per_step'],2), '%.3g'%d['value'], round(d['roofline']['achieved']), {k:round(v,2) for k,v in d['breakdown_ms'].items()})" || tail -3 gpurun_out/mode$m.err
  grep '\[owl\]' gpurun_out/mode$m.err | tail -2
done
if [ "${NCU:-1}" = "1" ]; then
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fold_kernel --launch-skip 2 -c 2 -o gpurun_out/prof_iter python bench.py --steps 1 --warmup 1 --no-cpu --no-e2e > gpurun_out/ncu_iter.log 2>&1
tail -1 gpurun_out/ncu_iter.log
fi
