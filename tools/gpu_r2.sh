#!/bin/bash
# One GPU session: all parity tests (incl. the H_cf R2 tests), smoke, one bench line.
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q --timeout 200 2>&1 | tail -25 > gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/bench.txt 2>gpurun_out/bench.err
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
