#!/bin/bash
# ncu launch list (gpu__time_duration only, clocks unlocked) of the C2 channel-order bench step (copy mode)
mkdir -p gpurun_out
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/co_launches.csv python bench.py --steps 1 --warmup 1 --no-cpu --no-e2e --channel-order ${BENCH_ARGS} > gpurun_out/co_launches.log 2>&1
tail -2 gpurun_out/co_launches.log
python tools/launch_summary.py gpurun_out/co_launches.csv > gpurun_out/co_launches.txt 2>&1; head -30 gpurun_out/co_launches.txt
