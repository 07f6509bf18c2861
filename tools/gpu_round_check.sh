#!/bin/bash
# Round-end style validation on one GPU: smoke, the GPU test suite, the default bench line,
# a 2-rank same-device run of the multi-rank path, and the f4 train bench.
set -u
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --out gpurun_out/bench_papers.json > gpurun_out/bench_papers.log 2>&1; echo bench=$?
GD_BENCH_SAME_DEVICE=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29511 bench.py --gpus 2 --steps 60 --warmup 4 --out gpurun_out/bench_papers_n2.json > gpurun_out/bench_papers_n2.log 2>&1
echo n2=$?
timeout 600 python bench.py --config products --train --steps 100 --no-cpu-baseline --parity-batches 0 \
    --out gpurun_out/bench_products_train.json > gpurun_out/bench_products_train.log 2>&1; echo train=$?
