mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -q -x --timeout 120 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
tail -2 gpurun_out/pytest_gpu.txt
for lib in libowl libowl_w24 libowl_w16; do
OWL_LIBOWL_PATH=$PWD/paper_conf_dsn_zhaoxcqzj24_b200/$lib.so OWL_FOLD_VERBOSE=1 timeout 300 python bench.py --steps 2 --warmup 1 --no-cpu --breakdown > gpurun_out/$lib.full.txt 2>gpurun_out/$lib.full.err
python -c "import json;d=json.loads(open('gpurun_out/$lib.full.txt').read().strip().splitlines()[-1]);print('$lib', round(d['ms_per_step'],1), '%.3g'%d['value'], round(d['roofline']['achieved']), {k:round(v,1) for k,v in d['breakdown_ms'].items()})" || tail -5 gpurun_out/$lib.full.err
grep owl gpurun_out/$lib.full.err | tail -2
done
