mkdir -p gpurun_out
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
for m in 2 1 0; do OWL_FOLD_MODE=$m timeout 300 python bench.py --steps 2 --warmup 1 --runs 40 --no-cpu > gpurun_out/mode$m.txt 2>&1; done
tail -3 gpurun_out/pytest_gpu.txt
for m in 2 1 0; do python -c "import json;d=json.loads(open('gpurun_out/mode$m.txt').read().strip().splitlines()[-1]);print($m, d['ms_per_step'], d['roofline']['achieved'], d['roofline']['note'][:60], d['fold_share_of_step'])" || tail -5 gpurun_out/mode$m.txt; done
