#!/bin/bash
# global address table sizing sweep (OWL_ADDR_LOAD_SHIFT: capacity = next_pow2(cells << shift)) on configs CFGS
mkdir -p gpurun_out
line() { python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);print(sys.argv[2], round(d['ms_per_step'],2), '%.3g'%d['value'], 'fold', round(d['roofline']['achieved']), 'frac', round(d['roofline']['frac'],3), d['clocks'].get('sm_mhz'))" $1 $2 || tail -5 ${1%.txt}.err; }
for cfg in ${CFGS:-2 3}; do
  for sh in ${SHIFTS:-2 3 4}; do
    OWL_ADDR_LOAD_SHIFT=$sh timeout 600 python bench.py --config $cfg --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/sh_c${cfg}_s$sh.txt 2> gpurun_out/sh_c${cfg}_s$sh.err; line gpurun_out/sh_c${cfg}_s$sh.txt c${cfg}_shift$sh
  done
done
