mkdir -p gpurun_out
timeout 600 ncu --set full --clock-control none --import-source on -k regex:fold_kernel -s 2 -c 1 -o gpurun_out/prof_full python bench.py --steps 1 --warmup 1 --runs 64 --no-cpu > gpurun_out/ncu_full.log 2>&1
tail -3 gpurun_out/ncu_full.log
