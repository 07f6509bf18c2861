# pop_assign loads-first + {pos,node} miss list, hash claim, relabel loads: parity + A/B + launch lists
set -u
mkdir -p gpurun_out/pop
python tools/build_native.py > /dev/null
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench.py -m gpu -q -x > gpurun_out/pop/pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pop/pytest.log
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for C in products papers100m mag240m friendster; do
    timeout 900 python bench.py --config $C $A > gpurun_out/pop/$C.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/pop/$C.json').readline());print('$C',d['value'],d['e2e']['value'],d['roofline']['frac'],d.get('roofline_gather',d['roofline'])['frac'])"
done
for C in products papers100m; do
timeout 900 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum --kernel-name-base function -k regex:'^k_' --csv --log-file gpurun_out/pop/${C}_warm.csv \
  python bench.py --config $C --steps 6 --warmup 3 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e > /dev/null 2>&1; echo ncu=$?
done
