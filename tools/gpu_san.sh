#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over tools/san_case.py (C1 full, C2 slices, config 9);
# summaries to gpurun_out/san_<tool>.txt
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  extra=""
  [ $tool = racecheck ] && extra="--racecheck-report hazard"
  timeout 1500 compute-sanitizer --tool $tool $extra --print-limit 200 python tools/san_case.py > gpurun_out/san_$tool.txt 2>&1
  echo "== $tool rc=$?"; grep -E "ERROR SUMMARY|RACECHECK SUMMARY|hazard|C[0-9] div" gpurun_out/san_$tool.txt | sort | uniq -c | head -20
done
