mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -q -x --timeout 120 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
tail -2 gpurun_out/pytest_gpu.txt
OWL_FOLD_VERBOSE=1 timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu --breakdown > gpurun_out/full.txt 2>gpurun_out/full.err
python -c "import json;d=json.loads(open('gpurun_out/full.txt').read().strip().splitlines()[-1]);print(round(d['ms_per_step'],1), '%.3g'%d['value'], round(d['roofline']['achieved']), {k:round(v,1) for k,v in d['breakdown_ms'].items()})" || tail -5 gpurun_out/full.err
grep owl gpurun_out/full.err | tail -2
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fold_kernel -s 2 -c 2 -o gpurun_out/prof_w24 python bench.py --steps 1 --warmup 1 --runs 64 --no-cpu > gpurun_out/ncu_w24.log 2>&1
tail -1 gpurun_out/ncu_w24.log
