#!/bin/bash
# ncu --set full of the FIX and RND fold launches of the first timed step (warmup 1 skipped) for each
# (name:lib:mode) in $CAPS; env passes through (OWL_ADDR_LOAD_SHIFT etc.).
mkdir -p gpurun_out
for c in $CAPS; do
  IFS=: read n l m <<< "$c"
  OWL_LIBOWL_PATH=paper_conf_dsn_zhaoxcqzj24_b200/$l OWL_FOLD_MODE=$m timeout 900 ncu --set full --clock-control none --import-source on -k regex:fold_kernel --launch-skip 2 -c 2 -o gpurun_out/prof_$n python bench.py --steps 1 --warmup 1 --no-cpu --no-e2e --runs ${RUNS:-40} > gpurun_out/prof_$n.log 2>&1
  tail -1 gpurun_out/prof_$n.log
done
