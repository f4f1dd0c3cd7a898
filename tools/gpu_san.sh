mkdir -p gpurun_out
timeout 600 compute-sanitizer --tool memcheck --show-backtrace device python -m pytest tests -m gpu -q -x -k "config_parity and 2-32" > gpurun_out/san.txt 2>&1
grep -m 20 -E "=========|Invalid|Illegal|at 0x|owl_fold" gpurun_out/san.txt | head -40
