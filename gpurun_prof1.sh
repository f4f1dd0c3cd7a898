mkdir -p gpurun_out
for m in 2 1 0; do OWL_FOLD_MODE=$m timeout 300 python bench.py --steps 2 --warmup 1 --runs 20 --no-cpu > gpurun_out/mode$m.txt 2>&1; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 0 --runs 20 --no-cpu > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fold_kernel -c 1 -o gpurun_out/prof_fold python bench.py --steps 1 --warmup 0 --runs 8 --no-cpu > gpurun_out/ncu_full.log 2>&1
for m in 2 1 0; do python -c "import json;d=json.loads(open('gpurun_out/mode$m.txt').read().strip().splitlines()[-1]);print($m, d['ms_per_step'], d['roofline']['achieved'], d['roofline']['note'])"; done
