#!/bin/bash
# One GPU session: parity tests, smoke, bench line (+ breakdown), ncu launch list, ncu full capture of the fold kernel.
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
timeout 600 python -m pytest tests -m gpu -q -x --timeout 200 2>&1 | tail -20 > gpurun_out/pytest_gpu.txt
tail -2 gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; tail -1 gpurun_out/smoke.txt
timeout 600 python bench.py --breakdown --no-cpu --no-e2e > gpurun_out/bench_brk.txt 2>gpurun_out/bench_brk.err; tail -c 600 gpurun_out/bench_brk.txt
timeout 900 python bench.py > gpurun_out/bench.txt 2>gpurun_out/bench.err; tail -c 1500 gpurun_out/bench.txt
timeout 300 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref.txt 2>gpurun_out/bench_ref.err; tail -c 400 gpurun_out/bench_ref.txt
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 0 --no-cpu --no-e2e > gpurun_out/launches.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fold_kernel --launch-skip 2 -c 1 -o gpurun_out/prof_fold python bench.py --steps 1 --warmup 1 --no-cpu --no-e2e > gpurun_out/ncu_full.log 2>&1
tail -1 gpurun_out/ncu_full.log
