# e2e vs device-timed region, per 50-step window (papers100m x2, default config)
set -u
mkdir -p gpurun_out/e2e
A="--config papers100m --no-cpu-baseline --parity-batches 0 --no-replay --window 50"
for i in 1 2 3; do
  timeout 900 python bench.py $A > gpurun_out/e2e/p_$i.json 2>/dev/null
  python -c "import json;d=json.loads(open('gpurun_out/e2e/p_$i.json').readline());print('papers',d['value'],d['e2e']['value'],d['roofline']['per_path_GBps']['host_gather_phase1']);print(' timed',d['windows']);print(' e2e',d['e2e']['windows'])"
done
