mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -q -x --timeout 120 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
tail -2 gpurun_out/pytest_gpu.txt
OWL_FOLD_VERBOSE=1 timeout 300 python bench.py --steps 2 --warmup 1 --no-cpu --breakdown > gpurun_out/full_brk.txt 2>gpurun_out/full_brk.err
python -c "import json;d=json.loads(open('gpurun_out/full_brk.txt').read().strip().splitlines()[-1]);print(d['ms_per_step'], d['value'], d['roofline']['achieved'], d['breakdown_ms'], d['result'])" || tail -5 gpurun_out/full_brk.err
grep owl gpurun_out/full_brk.err | tail -2
