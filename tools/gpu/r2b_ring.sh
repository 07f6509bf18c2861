# sample-ahead ring A/B (products, papers100m, tiny), then the GPU tests touching bench
set -u
mkdir -p gpurun_out/ring
python tools/build_native.py > /dev/null
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for C in products tiny; do
for R in 0 3 6 3 0; do
    timeout 600 python bench.py --config $C --sample-ahead $R $A > gpurun_out/ring/${C}_ra$R.json 2> gpurun_out/ring/${C}_ra$R.log
    python -c "import json;d=json.loads(open('gpurun_out/ring/${C}_ra$R.json').readline());print('$C ahead=$R',d['value'],d['e2e']['value'],d['per_batch']['sample_ms_per_batch'])"
done
done
for R in 0 3; do
    timeout 900 python bench.py --config papers100m --sample-ahead $R $A > gpurun_out/ring/papers_ra$R.json 2> gpurun_out/ring/papers_ra$R.log
    python -c "import json;d=json.loads(open('gpurun_out/ring/papers_ra$R.json').readline());print('papers ahead=$R',d['value'],d['e2e']['value'],d['roofline']['frac'])"
done
timeout 900 python bench.py --config products --samplers 3 $A > gpurun_out/ring/products_s3.json 2>/dev/null
python -c "import json;d=json.loads(open('gpurun_out/ring/products_s3.json').readline());print('products S3 ahead=3',d['value'],d['e2e']['value'])"
timeout 600 python bench.py --config products --steps 100 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e --timeline gpurun_out/ring/products_timeline.md > /dev/null 2>&1; echo tl=$?
timeout 1200 python -m pytest tests/test_gpu_bench.py -m gpu -q -x > gpurun_out/ring/pytest_bench.log 2>&1; echo pytest_bench=$?; tail -2 gpurun_out/ring/pytest_bench.log
