# the e2e gap: default papers100m line with and without the first-batch parity check (same box)
set -u
mkdir -p gpurun_out/e2e2
for P in 8 0 8 0; do
  timeout 900 python bench.py --config papers100m --parity-batches $P --no-cpu-baseline --no-replay > gpurun_out/e2e2/p$P.json 2>/dev/null
  python -c "import json;d=json.loads(open('gpurun_out/e2e2/p$P.json').readline());print('parity $P',d['value'],d['e2e']['value'],d['roofline']['per_path_GBps']['host_gather_phase1'])"
done
