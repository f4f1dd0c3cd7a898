#!/bin/bash
# Parity of the C2 config test under fold experiment modes (bisecting a fold failure).
mkdir -p gpurun_out
for m in ${MODES:-0 9 10}; do
  OWL_FOLD_MODE=$m timeout 120 python -m pytest tests -m gpu -q -x -k "config_parity and 2-32" 2>&1 | grep -E "Error|error|assert|passed|failed" | head -5 | sed "s/^/mode $m: /"
done
