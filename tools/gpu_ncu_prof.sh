#!/bin/bash
# ncu --set full of one steady-state fold launch (FIX class, full C2 workload) for each lib in $LIBS
# (name:path), summaries into gpurun_out/<name>_ncu.txt (+ per-source-line shares).
mkdir -p gpurun_out
for spec in $LIBS; do
  n=${spec%%:*}; lib=${spec#*:}
  OWL_LIBOWL_PATH=$lib timeout 900 ncu --set full --clock-control none --import-source on -k regex:fold_kernel --launch-skip 2 -c 1 -o gpurun_out/prof_$n python bench.py --steps 1 --warmup 1 --no-cpu --no-e2e > gpurun_out/prof_$n.log 2>&1
  ncu -i gpurun_out/prof_$n.ncu-rep --page raw --csv > gpurun_out/prof_$n.raw.csv 2>/dev/null
  python tools/ncu_summary.py gpurun_out/prof_$n.raw.csv 1391820800 > gpurun_out/${n}_ncu.txt
  ncu -i gpurun_out/prof_$n.ncu-rep --page source --csv --print-source cuda,sass > gpurun_out/prof_$n.src.csv 2>/dev/null
  python tools/ncu_lines.py gpurun_out/prof_$n.src.csv 45 > gpurun_out/${n}_lines.txt 2>&1
  head -30 gpurun_out/${n}_ncu.txt
done
