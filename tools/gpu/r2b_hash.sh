# double-buffered relabel hash (previous call's table emptied inside the last relabel pass): parity + A/B
set -u
mkdir -p gpurun_out/hash
python tools/build_native.py > /dev/null
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench.py tests/test_gpu_train.py -m gpu -q -x > gpurun_out/hash/pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/hash/pytest.log
GD_HASH_CLEAR_KERNEL=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k sample > gpurun_out/hash/pytest_k.log 2>&1; echo pytest_clear_kernel=$?; tail -1 gpurun_out/hash/pytest_k.log
python -c "import __graft_entry__ as g; g.smoke()"; echo smoke=$?
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for C in products tiny; do
for K in 0 1 0 1; do
    GD_HASH_CLEAR_KERNEL=$K timeout 600 python bench.py --config $C $A > gpurun_out/hash/${C}_k$K.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/hash/${C}_k$K.json').readline());print('$C clear_kernel=$K',d['value'],d['e2e']['value'],d['roofline']['frac'])"
done
done
timeout 900 python bench.py --config products --parity-batches 16 --no-cpu-baseline > gpurun_out/hash/products_parity.json 2>/dev/null; echo products_parity=$?
python -c "import json;d=json.loads(open('gpurun_out/hash/products_parity.json').readline());print(d['value'], d['parity']['bit_exact'], d['parity']['steady_state']['batches'])"
timeout 900 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --kernel-name-base function -k regex:'^k_' --csv --log-file gpurun_out/hash/products_warm.csv \
  python bench.py --config products --steps 6 --warmup 3 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e > /dev/null 2>&1; echo ncu=$?
