#!/bin/bash
# Like gpu_var.sh but fold-only numbers (no breakdown syncs), plus mode-2 skeleton of the default lib.
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -q -x --timeout 60 2>&1 | tail -3 > gpurun_out/pytest_gpu.txt
tail -1 gpurun_out/pytest_gpu.txt
for lib in ${LIBS:-libowl}; do
 for m in ${MODES:-0}; do
  OWL_LIBOWL_PATH=$PWD/paper_conf_dsn_zhaoxcqzj24_b200/$lib.so OWL_FOLD_MODE=$m OWL_FOLD_VERBOSE=1 timeout 150 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e > gpurun_out/$lib.m$m.txt 2> gpurun_out/$lib.m$m.err
  python -c "import json;d=json.loads(open('gpurun_out/$lib.m$m.txt').read().strip().splitlines()[-1]);print('$lib mode $m step', round(d['ms_per_step'],2), 'rec/s %.3g'%d['value'], 'fold GB/s', round(d['roofline']['achieved']))" || tail -3 gpurun_out/$lib.m$m.err
  grep '\[owl\]' gpurun_out/$lib.m$m.err | tail -3 | head -2
 done
done
