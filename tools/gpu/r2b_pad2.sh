# padded sampler v2 (col resolved in k_relabel_pad): parity, A/B, launch lists, timelines
set -u
mkdir -p gpurun_out/pad2
python tools/build_native.py > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "sample" > gpurun_out/pad2/pytest_sample.log 2>&1; echo pytest_sample=$?; tail -2 gpurun_out/pad2/pytest_sample.log
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for S in 2 3 4; do
for P in 1 0; do
    GD_SAMPLE_PAD=$P timeout 600 python bench.py --config products --samplers $S $A > gpurun_out/pad2/products_s${S}_pad$P.json 2> gpurun_out/pad2/products_s${S}_pad$P.log
    python -c "import json;d=json.loads(open('gpurun_out/pad2/products_s${S}_pad$P.json').readline());print('products S=$S pad=$P',d['value'],d['e2e']['value'],d['per_batch']['sample_ms_per_batch'])"
done
done
GD_SAMPLE_PAD=1 timeout 900 python bench.py --config products --parity-batches 16 --no-cpu-baseline > gpurun_out/pad2/products_parity.json 2> gpurun_out/pad2/products_parity.log; echo products_parity=$?
python -c "import json;d=json.loads(open('gpurun_out/pad2/products_parity.json').readline());print(d['value'], json.dumps(d['parity'])[:300])"
GD_SAMPLE_PAD=1 timeout 900 python bench.py --config papers100m --parity-batches 8 --no-cpu-baseline > gpurun_out/pad2/papers_parity.json 2> gpurun_out/pad2/papers_parity.log; echo papers_parity=$?
python -c "import json;d=json.loads(open('gpurun_out/pad2/papers_parity.json').readline());print(d['value'], d['roofline']['frac'], json.dumps(d['parity'])[:300])"
for P in 1 0; do
GD_SAMPLE_PAD=$P timeout 600 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum --kernel-name-base function -k regex:'^k_' --csv --log-file gpurun_out/pad2/products_warm_pad$P.csv \
  python bench.py --config products --steps 6 --warmup 3 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e > /dev/null 2>&1; echo ncu=$?
GD_SAMPLE_PAD=$P timeout 600 python bench.py --config products --steps 100 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e --timeline gpurun_out/pad2/products_timeline_pad$P.md > /dev/null 2>&1; echo tl=$?
done
