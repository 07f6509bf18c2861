set -u
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1200 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --out gpurun_out/bench_papers.json > gpurun_out/bench_papers.log 2>&1; echo bench=$?
timeout 600 python bench.py --config papers100m --train --steps 100 --no-cpu-baseline --parity-batches 0 --out gpurun_out/bench_papers_train.json > gpurun_out/bench_papers_train.log 2>&1; echo train_papers=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:umma -c 3 -o gpurun_out/prof_umma_products -f python bench.py --config products --train --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --parity-batches 0 --prewarm-max 8 > gpurun_out/ncu_umma_products.log 2>&1; echo ncu=$?
