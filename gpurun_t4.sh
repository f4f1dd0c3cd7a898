mkdir -p gpurun_out
timeout 400 python -m pytest tests -m gpu -q -x --timeout 120 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
tail -2 gpurun_out/pytest_gpu.txt
for m in 3 2 1 0; do OWL_FOLD_VERBOSE=1 OWL_FOLD_MODE=$m timeout 120 python bench.py --steps 2 --warmup 1 --runs 40 --no-cpu > gpurun_out/mode$m.txt 2>gpurun_out/mode$m.err;
python -c "import json;d=json.loads(open('gpurun_out/mode$m.txt').read().strip().splitlines()[-1]);print($m, round(d['ms_per_step'],2), round(d['roofline']['achieved']), d['roofline']['note'][:60], round(d['fold_share_of_step'],3))" || tail -3 gpurun_out/mode$m.txt; tail -2 gpurun_out/mode$m.err; done
