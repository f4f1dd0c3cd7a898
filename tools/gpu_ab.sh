#!/bin/bash
# A/B iteration on one box: GPU parity tests on the product library, then bench (fold mode 0 and the
# stream-only mode 2) for the product library and every variant library named in $VARIANTS.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
if [ "${TESTS:-1}" = "1" ]; then
  timeout 600 python -m pytest tests -m gpu -q -x --timeout 200 2>&1 | tail -20 > gpurun_out/pytest_gpu.txt
  tail -3 gpurun_out/pytest_gpu.txt
fi
run() { # name lib mode
  OWL_LIBOWL_PATH=$2 OWL_FOLD_MODE=$3 OWL_FOLD_VERBOSE=1 timeout 300 python bench.py --steps ${STEPS:-3} --warmup 2 --no-cpu --no-e2e --breakdown > gpurun_out/ab_$1_m$3.txt 2> gpurun_out/ab_$1_m$3.err
  python -c "import json;d=json.loads(open('gpurun_out/ab_$1_m$3.txt').read().strip().splitlines()[-1]);print('$1 mode $3', round(d['ms_per_step'],2), '%.3g'%d['value'], round(d['roofline']['achieved']), {k:round(v,2) for k,v in d['breakdown_ms'].items()})" || tail -5 gpurun_out/ab_$1_m$3.err
  grep '\[owl\]' gpurun_out/ab_$1_m$3.err | tail -2
}
run prod paper_conf_dsn_zhaoxcqzj24_b200/libowl.so 0
run prod paper_conf_dsn_zhaoxcqzj24_b200/libowl.so 2
for v in $VARIANTS; do run $v paper_conf_dsn_zhaoxcqzj24_b200/libowl_$v.so ${VMODE:-0}; done
for m in $MODES; do run prod paper_conf_dsn_zhaoxcqzj24_b200/libowl.so $m; done
