#!/bin/bash
# ncu --set full of one steady-state fold launch of bench config $CFG (default 2), summary + source lines.
mkdir -p gpurun_out
CFG=${CFG:-2}; n=${NAME:-c$CFG}
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:fold_kernel --launch-skip ${SKIP:-2} -c 1 -o gpurun_out/prof_$n python bench.py --config $CFG --steps 1 --warmup 1 --no-cpu --no-e2e ${ARGS} > gpurun_out/prof_$n.log 2>&1
ncu -i gpurun_out/prof_$n.ncu-rep --page raw --csv > gpurun_out/prof_$n.raw.csv 2>/dev/null
python tools/ncu_summary.py gpurun_out/prof_$n.raw.csv ${RECS:-} > gpurun_out/${n}_ncu.txt
ncu -i gpurun_out/prof_$n.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/prof_$n.src.csv 2>/dev/null
python tools/ncu_lines.py gpurun_out/prof_$n.src.csv 45 > gpurun_out/${n}_lines.txt 2>&1
head -24 gpurun_out/${n}_ncu.txt
