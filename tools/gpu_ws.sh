#!/bin/bash
# warp-specialized fold (OWL_FOLD_WS=1): GPU tests, then C2 bench lines for prod vs WS variants (VARS)
mkdir -p gpurun_out
if [ "${TESTS:-1}" = "1" ]; then
  OWL_FOLD_WS=1 timeout 900 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS} 2>&1 | tail -30 > gpurun_out/pytest_gpu_ws.txt
  tail -4 gpurun_out/pytest_gpu_ws.txt
fi
line() { python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);print(sys.argv[2], round(d['ms_per_step'],2), '%.3g'%d['value'], 'fold', round(d['roofline']['achieved']), 'frac', round(d['roofline']['frac'],3), d['clocks'].get('sm_mhz'))" $1 $2 || tail -5 ${1%.txt}.err; }
for cfg in ${CFGS:-2}; do
  OWL_FOLD_VERBOSE=1 timeout 400 python bench.py --config $cfg --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/ws_prod_c$cfg.txt 2> gpurun_out/ws_prod_c$cfg.err; line gpurun_out/ws_prod_c$cfg.txt prod_c$cfg
  for v in $VARS; do
    if [ "$v" = "ws" ]; then lib=paper_conf_dsn_zhaoxcqzj24_b200/libowl.so; else lib=paper_conf_dsn_zhaoxcqzj24_b200/libowl_$v.so; fi
    OWL_LIBOWL_PATH=$lib OWL_FOLD_WS=1 OWL_FOLD_VERBOSE=1 timeout 400 python bench.py --config $cfg --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/ws_${v}_c$cfg.txt 2> gpurun_out/ws_${v}_c$cfg.err; line gpurun_out/ws_${v}_c$cfg.txt ${v}_c$cfg; grep '\[owl\]' gpurun_out/ws_${v}_c$cfg.err | tail -1
  done
done
if [ -n "$NCUWS" ]; then
OWL_FOLD_WS=1 timeout 900 ncu --set full --clock-control none --import-source on -k regex:fold_ws_kernel --launch-skip 2 -c 1 -o gpurun_out/prof_ws python bench.py --steps 1 --warmup 2 --no-cpu --no-e2e > gpurun_out/ncu_ws.log 2>&1; tail -1 gpurun_out/ncu_ws.log
fi
