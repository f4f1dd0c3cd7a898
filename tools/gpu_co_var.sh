#!/bin/bash
# C2 channel-order bench lines, repeated (variance check), full contract and --no-cpu --no-e2e
mkdir -p gpurun_out
line() { python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);print(sys.argv[2], round(d['ms_per_step'],2), '%.3g'%d['value'], 'fold', round(d['roofline']['achieved']), d['config'].get('record_order'))" $1 $2 || tail -5 ${1%.txt}.err; }
for k in 1 2; do
  OWL_FOLD_VERBOSE=1 timeout 900 python bench.py --channel-order --steps 5 --warmup 3 > gpurun_out/cov_full_$k.txt 2> gpurun_out/cov_full_$k.err; line gpurun_out/cov_full_$k.txt full_$k
  timeout 900 python bench.py --channel-order --steps 5 --warmup 3 --no-cpu --no-e2e > gpurun_out/cov_lite_$k.txt 2> gpurun_out/cov_lite_$k.err; line gpurun_out/cov_lite_$k.txt lite_$k
done
