#!/bin/bash
# ncu --set full of the two fold launches of one bench step (FIX, RND); OWL_LIBOWL_PATH / OWL_FOLD_MODE honoured.
mkdir -p gpurun_out
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fold_kernel -c 2 -o gpurun_out/${PROF:-prof} python bench.py --steps 1 --warmup 0 --no-cpu > gpurun_out/${PROF:-prof}.log 2>&1
tail -1 gpurun_out/${PROF:-prof}.log
