# dirty-tracked tile-state clears: parity, products / papers rates, warm launch list
set -u
mkdir -p gpurun_out/clr
python tools/build_native.py > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench.py -m gpu -q -x > gpurun_out/clr/pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/clr/pytest.log
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for C in products products tiny papers100m; do
    timeout 900 python bench.py --config $C $A > gpurun_out/clr/$C.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/clr/$C.json').readline());print('$C',d['value'],d['e2e']['value'],d['roofline']['frac'],d.get('roofline_gather',d['roofline'])['frac'])"
done
timeout 900 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum --kernel-name-base function -k regex:'^k_' --csv --log-file gpurun_out/clr/products_warm.csv \
  python bench.py --config products --steps 6 --warmup 3 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e > /dev/null 2>&1; echo ncu=$?
