mkdir -p gpurun_out
for ls in 1 2 3 4; do
  OWL_ADDR_LOAD_SHIFT=$ls timeout 300 python bench.py --steps 3 --warmup 2 --no-cpu --no-e2e --breakdown > gpurun_out/ls$ls.txt 2> gpurun_out/ls$ls.err
  python -c "import json;d=json.loads(open('gpurun_out/ls$ls.txt').read().strip().splitlines()[-1]);print('load_shift $ls', round(d['ms_per_step'],2), '%.3g'%d['value'], {k:round(v,2) for k,v in d['breakdown_ms'].items()})" || tail -3 gpurun_out/ls$ls.err
done
