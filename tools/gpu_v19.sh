#!/bin/bash
# v19 fold A/B: GPU tests against the variant lib, then bench lines for prod and the variant on C2 (and C3-C5 if CFGS).
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader > gpurun_out/smi.txt 2>&1
V=${V:-v19}
if [ "${TESTS:-1}" = "1" ]; then
  OWL_LIBOWL_PATH=paper_conf_dsn_zhaoxcqzj24_b200/libowl_$V.so timeout 900 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS} 2>&1 | tail -30 > gpurun_out/pytest_gpu_$V.txt
  tail -4 gpurun_out/pytest_gpu_$V.txt
fi
run() { # name lib mode cfg
  OWL_LIBOWL_PATH=$2 OWL_FOLD_MODE=$3 OWL_FOLD_VERBOSE=1 timeout 400 python bench.py --config $4 --steps ${STEPS:-5} --warmup 3 --no-cpu --no-e2e ${BENCH_ARGS} > gpurun_out/ab_$1_m$3_c$4.txt 2> gpurun_out/ab_$1_m$3_c$4.err
  python -c "import json;d=json.loads(open('gpurun_out/ab_$1_m$3_c$4.txt').read().strip().splitlines()[-1]);print('$1 mode $3 cfg $4', round(d['ms_per_step'],2), '%.3g'%d['value'], 'fold', round(d['roofline']['achieved']), 'GB/s frac', round(d['roofline']['frac'],3), d['clocks'].get('sm_mhz'))" || tail -5 gpurun_out/ab_$1_m$3_c$4.err
  grep '\[owl\]' gpurun_out/ab_$1_m$3_c$4.err | tail -2
}
for spec in $RUNS; do  # name:mode:cfg
  n=${spec%%:*}; rest=${spec#*:}; m=${rest%%:*}; c=${rest#*:}
  if [ "$n" = "prod" ]; then lib=paper_conf_dsn_zhaoxcqzj24_b200/libowl.so; else lib=paper_conf_dsn_zhaoxcqzj24_b200/libowl_$n.so; fi
  run $n $lib $m $c
done
