set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,memory.total,clocks.sm,clocks.max.sm --format=csv > gpurun_out/box.txt 2>&1
free -g >> gpurun_out/box.txt; nproc >> gpurun_out/box.txt; lscpu | grep "Model name" >> gpurun_out/box.txt
timeout 900 python -m pytest tests -m gpu -q -x --timeout 600 2>&1 | tail -40 > gpurun_out/pytest_gpu.txt
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.txt 2>&1
timeout 600 python bench.py --steps 2 --warmup 1 --runs 20 --no-cpu > gpurun_out/bench_small.txt 2>&1
tail -5 gpurun_out/pytest_gpu.txt
cat gpurun_out/smoke.txt | tail -5
cat gpurun_out/bench_small.txt | tail -5
