#!/bin/bash
# A/B on one box: GPU tests (TESTS=1), then `run name lib mode` bench lines for the product and variant libs.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader > gpurun_out/smi.txt 2>&1
if [ "${TESTS:-1}" = "1" ]; then
  timeout 900 python -m pytest tests -m gpu -q ${PYTEST_ARGS:--x} 2>&1 | tail -25 > gpurun_out/pytest_gpu.txt
  tail -4 gpurun_out/pytest_gpu.txt
fi
run() { # name lib mode
  OWL_LIBOWL_PATH=$2 OWL_FOLD_MODE=$3 OWL_FOLD_VERBOSE=1 timeout 300 python bench.py --steps ${STEPS:-5} --warmup 3 --no-cpu --no-e2e ${BENCH_ARGS} > gpurun_out/ab_$1_m$3.txt 2> gpurun_out/ab_$1_m$3.err
  python -c "import json;d=json.loads(open('gpurun_out/ab_$1_m$3.txt').read().strip().splitlines()[-1]);print('$1 mode $3', round(d['ms_per_step'],2), '%.3g'%d['value'], 'fold', round(d['roofline']['achieved']), 'GB/s frac', round(d['roofline']['frac'],3), d['clocks'].get('sm_mhz'))" || tail -5 gpurun_out/ab_$1_m$3.err
  grep '\[owl\]' gpurun_out/ab_$1_m$3.err | tail -1
}
for spec in $RUNS; do  # name:mode (lib = libowl_<name>.so, name "prod" = libowl.so)
  n=${spec%%:*}; m=${spec#*:}
  if [ "$n" = "prod" ]; then lib=paper_conf_dsn_zhaoxcqzj24_b200/libowl.so; else lib=paper_conf_dsn_zhaoxcqzj24_b200/libowl_$n.so; fi
  run $n $lib $m
done
