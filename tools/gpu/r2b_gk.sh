# hoisted lookup/release loads: parity; gather grid / rows-in-flight A/B; warm launch list
set -u
mkdir -p gpurun_out/gk
python tools/build_native.py > /dev/null
timeout 1200 python -m pytest tests/test_gpu_parity.py -m gpu -q -x > gpurun_out/gk/pytest_parity.log 2>&1; echo pytest_parity=$?; tail -2 gpurun_out/gk/pytest_parity.log
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for V in 4:4 2:8 3:8 4:8 6:4 4:4; do
    B=${V%:*}; U=${V#*:}
    GD_GATHER_BPS=$B GD_GATHER_U=$U timeout 600 python bench.py --config products $A > gpurun_out/gk/products_${B}_${U}.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/gk/products_${B}_${U}.json').readline());print('products bps=$B U=$U',d['value'],d['e2e']['value'],d['roofline']['frac'],d['roofline']['isolated']['frac'])"
done
for V in 4:4 2:8; do
    B=${V%:*}; U=${V#*:}
    GD_GATHER_BPS=$B GD_GATHER_U=$U timeout 900 python bench.py --config papers100m $A > gpurun_out/gk/papers_${B}_${U}.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/gk/papers_${B}_${U}.json').readline());print('papers bps=$B U=$U',d['value'],d['e2e']['value'],d['roofline']['frac'],d['roofline_gather']['frac'],d['roofline_gather']['isolated']['frac'])"
done
timeout 600 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum --kernel-name-base function -k regex:'^k_' --csv --log-file gpurun_out/gk/products_warm.csv \
  python bench.py --config products --steps 6 --warmup 3 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e > /dev/null 2>&1; echo ncu=$?
