# padded sampler: parity (both variants), products / tiny / papers100m A/B, warm launch list
set -u
mkdir -p gpurun_out/pad
python tools/build_native.py > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "sample" > gpurun_out/pad/pytest_sample.log 2>&1; echo pytest_sample=$?; tail -2 gpurun_out/pad/pytest_sample.log
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for C in products tiny; do
  for P in 1 0 1 0; do
    GD_SAMPLE_PAD=$P timeout 600 python bench.py --config $C $A > gpurun_out/pad/${C}_pad$P.json 2> gpurun_out/pad/${C}_pad$P.log
    python -c "import json;d=json.loads(open('gpurun_out/pad/${C}_pad$P.json').readline());print('$C pad=$P',d['value'],d['e2e']['value'],d['per_batch']['sample_ms_per_batch'])"
  done
done
GD_SAMPLE_PAD=1 timeout 900 python bench.py --config products --parity-batches 16 --no-cpu-baseline > gpurun_out/pad/products_parity.json 2> gpurun_out/pad/products_parity.log; echo products_parity=$?
python -c "import json;d=json.loads(open('gpurun_out/pad/products_parity.json').readline());print(d['value'], json.dumps(d['parity'])[:600])"
timeout 600 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum -k regex=k_ --csv --log-file gpurun_out/pad/products_warm.csv \
  python bench.py --config products --steps 6 --warmup 3 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e > /dev/null 2>&1; echo ncu=$?
