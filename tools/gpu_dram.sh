#!/bin/bash
# DRAM bytes of one steady-state fold launch under experiment modes (0 full, 1 no global table, 2 stream + walk).
# Needs a -DFOLD_RUNTIME_MODE build: tools/build_variant.sh rtmode "-DFOLD_RUNTIME_MODE"; OWL_LIBOWL_PATH=.../libowl_rtmode.so
mkdir -p gpurun_out
for m in ${MODES:-0 1 2}; do
  OWL_FOLD_MODE=$m timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read_evict_first_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_read_evict_normal_lookup_miss.sum,lts__t_sectors_srcunit_tex_op_read_evict_normal.sum --clock-control none -k regex:fold_kernel --launch-skip 2 -c 1 --csv python bench.py --steps 1 --warmup 1 --no-cpu --no-e2e 2>/dev/null | grep -E '"(gpu__time|dram__|lts__)' | awk -F'","' -v m=$m '{print "mode " m ": " $(NF-2) " " $(NF-1) " " $NF}'
done
