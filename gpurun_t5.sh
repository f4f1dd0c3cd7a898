mkdir -p gpurun_out
OWL_FOLD_VERBOSE=1 timeout 120 python bench.py --steps 2 --warmup 1 --runs 40 --no-cpu --breakdown > gpurun_out/brk.txt 2>gpurun_out/brk.err
python -c "import json;d=json.loads(open('gpurun_out/brk.txt').read().strip().splitlines()[-1]);print(d['ms_per_step'], d['breakdown_ms'])"
OWL_FOLD_MODE=2 timeout 300 ncu --set full --clock-control none -k regex:fold_kernel -c 1 -o gpurun_out/prof_m2 python bench.py --steps 1 --warmup 0 --runs 8 --no-cpu > gpurun_out/ncu2.log 2>&1
timeout 300 ncu --set full --clock-control none --import-source on -k regex:fold_kernel -s 1 -c 1 -o gpurun_out/prof_m0 python bench.py --steps 1 --warmup 0 --runs 8 --no-cpu > gpurun_out/ncu0.log 2>&1
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 0 --runs 40 --no-cpu > /dev/null 2>&1
ls gpurun_out
