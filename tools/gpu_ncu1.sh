#!/bin/bash
# ncu --set full of one steady-state fold launch (FIX class, full C2 workload), optional OWL_FOLD_MODE.
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fold_kernel --launch-skip 2 -c 1 -o gpurun_out/${PROF:-prof1} python bench.py --steps 1 --warmup 1 --no-cpu --no-e2e > gpurun_out/${PROF:-prof1}.log 2>&1
tail -1 gpurun_out/${PROF:-prof1}.log
