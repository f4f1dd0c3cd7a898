#!/bin/bash
# Round-end evidence on one B200: GPU test suite, smoke, default bench line (both arms), the ncu launch list of the
# bench command and one `ncu --set full` capture of a steady-state fold launch (C2, FIX class).
# Outputs under gpurun_out/final_*.
mkdir -p gpurun_out
o=gpurun_out/final
timeout 1500 python -m pytest tests -m gpu -q --timeout 900 -p no:cacheprovider > ${o}_pytest_gpu.txt 2>&1
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > ${o}_smoke.txt 2>&1
timeout 900 python bench.py > ${o}_bench.json 2>${o}_bench.err
timeout 900 python bench.py --impl reference > ${o}_bench_reference.json 2>${o}_bench_reference.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 6000 --csv --log-file ${o}_launches.csv \
  python bench.py --steps 1 --warmup 3 --no-cpu --no-e2e > ${o}_launches.log 2>&1
python tools/launch_summary.py ${o}_launches.csv > ${o}_launches.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:fold_kernel --launch-skip 2 -c 1 \
  -o ${o}_fold python bench.py --steps 1 --warmup 3 --no-cpu --no-e2e > ${o}_fold.log 2>&1
ncu -i ${o}_fold.ncu-rep --page raw --csv > ${o}_fold.raw.csv 2>/dev/null
python tools/ncu_summary.py ${o}_fold.raw.csv 1391820800 > ${o}_fold_ncu.txt 2>&1
ncu -i ${o}_fold.ncu-rep --page source --csv --print-source cuda,sass > ${o}_fold.src.csv 2>/dev/null
python tools/ncu_lines.py ${o}_fold.src.csv 45 > ${o}_fold_lines.txt 2>&1
rm -f ${o}_fold.src.csv
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > ${o}_smi.txt 2>&1
timeout 900 python bench.py --channel-order --steps 5 --warmup 3 > ${o}_bench_c2_channel.json 2>${o}_bench_c2_channel.err
timeout 900 python bench.py --channel-order --channel-mode inplace --steps 5 --warmup 3 > ${o}_bench_c2_channel_inplace.json 2>${o}_bench_c2_channel_inplace.err
