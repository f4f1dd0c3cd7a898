#!/bin/bash
# GPU test suite, then bench lines (no cpu / e2e legs) for the configs in CFGS and C2 channel order
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -30 > gpurun_out/pytest_gpu_all.txt; tail -3 gpurun_out/pytest_gpu_all.txt
line() { python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);print(sys.argv[2], round(d['ms_per_step'],2), '%.3g'%d['value'], 'fold', round(d['roofline']['achieved']), 'frac', round(d['roofline']['frac'],3), d['clocks'].get('sm_mhz'))" $1 $2 || tail -5 ${1%.txt}.err; }
for cfg in ${CFGS:-2 3 4 5}; do
  timeout 900 python bench.py --config $cfg --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/all_c$cfg.txt 2> gpurun_out/all_c$cfg.err; line gpurun_out/all_c$cfg.txt c$cfg
done
timeout 900 python bench.py --channel-order --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/all_co.txt 2> gpurun_out/all_co.err; line gpurun_out/all_co.txt c2-channel
