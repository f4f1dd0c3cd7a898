#!/bin/bash
# N2 in-place channel order: GPU tests, then C2 bench lines warp-major / channel order in place / channel order copy.
mkdir -p gpurun_out
if [ "${TESTS:-1}" = "1" ]; then
  timeout 900 python -m pytest tests -m gpu -q -x ${PYTEST_ARGS} 2>&1 | tail -30 > gpurun_out/pytest_gpu_n2.txt
  tail -4 gpurun_out/pytest_gpu_n2.txt
fi
line() { python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);print(sys.argv[2], round(d['ms_per_step'],2), '%.3g'%d['value'], 'fold', round(d['roofline']['achieved']), 'frac', round(d['roofline']['frac'],3), d['clocks'].get('sm_mhz'))" $1 $2 || tail -5 ${1%.txt}.err; }
OWL_FOLD_VERBOSE=1 timeout 400 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --breakdown > gpurun_out/n2_wm.txt 2> gpurun_out/n2_wm.err; line gpurun_out/n2_wm.txt warp-major; grep '\[owl\]' gpurun_out/n2_wm.err | tail -1
OWL_FOLD_VERBOSE=1 timeout 400 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --channel-order --channel-mode inplace --breakdown > gpurun_out/n2_ip.txt 2> gpurun_out/n2_ip.err; line gpurun_out/n2_ip.txt in-place; grep '\[owl\]' gpurun_out/n2_ip.err | tail -1
OWL_FOLD_VERBOSE=1 timeout 400 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --channel-order --channel-mode auto --breakdown > gpurun_out/n2_cp.txt 2> gpurun_out/n2_cp.err; line gpurun_out/n2_cp.txt copy; grep '\[owl\]' gpurun_out/n2_cp.err | tail -1
python - <<'PY'
import json
for f in ['n2_wm','n2_ip','n2_cp']:
    try:
        d=json.loads(open('gpurun_out/%s.txt'%f).read().strip().splitlines()[-1]); print(f, d.get('breakdown_ms'))
    except Exception as e: print(f, e)
PY
