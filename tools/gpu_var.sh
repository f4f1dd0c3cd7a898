#!/bin/bash
# Compare fold variants (libowl*.so) on the bench workload; modes 0 (full) and 2 (stream only).
mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -q -x --timeout 60 2>&1 | tail -3 > gpurun_out/pytest_gpu.txt
tail -2 gpurun_out/pytest_gpu.txt
for lib in ${LIBS:-libowl}; do
 for m in ${MODES:-0 2}; do
  OWL_LIBOWL_PATH=$PWD/paper_conf_dsn_zhaoxcqzj24_b200/$lib.so OWL_FOLD_MODE=$m OWL_FOLD_VERBOSE=1 timeout 150 python bench.py --steps 3 --warmup 2 --no-cpu --breakdown > gpurun_out/$lib.m$m.txt 2> gpurun_out/$lib.m$m.err
  python -c "import json;d=json.loads(open('gpurun_out/$lib.m$m.txt').read().strip().splitlines()[-1]);print('$lib mode $m', round(d['ms_per_step'],2), '%.3g'%d['value'], round(d['roofline']['achieved']), {k:round(v,2) for k,v in d['breakdown_ms'].items()})" || tail -3 gpurun_out/$lib.m$m.err
  grep '\[owl\]' gpurun_out/$lib.m$m.err | tail -2
 done
done
