#!/bin/bash
# ncu --set full of one steady-state fold launch of bench.py (C2 unless CFG) with a variant lib (V=name).
mkdir -p gpurun_out
V=${V:-v19}; CFG=${CFG:-2}
OWL_LIBOWL_PATH=paper_conf_dsn_zhaoxcqzj24_b200/libowl_$V.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:fold_kernel --launch-skip 2 -c 1 -o gpurun_out/prof_${V}_c$CFG python bench.py --config $CFG --steps 1 --warmup 2 --no-cpu --no-e2e > gpurun_out/ncu_${V}_c$CFG.log 2>&1
tail -2 gpurun_out/ncu_${V}_c$CFG.log
