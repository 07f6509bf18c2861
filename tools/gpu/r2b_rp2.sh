# relabel_pad: loads of all items before the dependent stores; clear loop 4 slots per round
set -u
mkdir -p gpurun_out/rp2
python tools/build_native.py > /dev/null
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_bench.py -m gpu -q -x > gpurun_out/rp2/pytest.log 2>&1; echo pytest=$?; tail -1 gpurun_out/rp2/pytest.log
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for C in products products papers100m; do
    timeout 900 python bench.py --config $C $A > gpurun_out/rp2/$C.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/rp2/$C.json').readline());print('$C',d['value'],d['e2e']['value'],d['roofline']['frac'],d['host_loop']['busy_ms_per_step'])"
done
timeout 900 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --kernel-name-base function -k regex:'^k_' --csv --log-file gpurun_out/rp2/products_warm.csv \
  python bench.py --config products --steps 6 --warmup 3 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e > /dev/null 2>&1; echo ncu=$?
python tools/launch_table.py gpurun_out/rp2/products_warm.csv | head -8
