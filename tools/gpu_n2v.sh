#!/bin/bash
# channel-order C2 bench lines for variant libs (VARS="name ..."), then an ncu capture of the in-place fold (NCUV)
mkdir -p gpurun_out
line() { python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);print(sys.argv[2], round(d['ms_per_step'],2), '%.3g'%d['value'], 'fold', round(d['roofline']['achieved']), 'frac', round(d['roofline']['frac'],3), d['clocks'].get('sm_mhz'))" $1 $2 || tail -5 ${1%.txt}.err; }
for v in $VARS; do
  OWL_LIBOWL_PATH=paper_conf_dsn_zhaoxcqzj24_b200/libowl_$v.so OWL_FOLD_VERBOSE=1 timeout 400 python bench.py --steps 5 --warmup 3 --no-cpu --no-e2e --channel-order ${BENCH_ARGS} > gpurun_out/n2v_$v.txt 2> gpurun_out/n2v_$v.err; line gpurun_out/n2v_$v.txt $v; grep '\[owl\]' gpurun_out/n2v_$v.err | tail -1
done
if [ -n "$NCUV" ]; then
OWL_LIBOWL_PATH=paper_conf_dsn_zhaoxcqzj24_b200/libowl_$NCUV.so timeout 900 ncu --set full --clock-control none --import-source on -k regex:fold_burst_kernel --launch-skip 2 -c 1 -o gpurun_out/prof_n2_$NCUV python bench.py --steps 1 --warmup 2 --no-cpu --no-e2e --channel-order > gpurun_out/ncu_n2_$NCUV.log 2>&1; tail -1 gpurun_out/ncu_n2_$NCUV.log
fi
