set -u
python tools/build_native.py > /dev/null
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu5.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu5.log
for r in 1 2 3; do
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/drv$r.json 2> gpurun_out/drv$r.err; echo "drv$r rc=$?"
done
timeout 900 python bench.py --config mag240m --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/drv_mag.json 2> gpurun_out/drv_mag.err; echo "mag rc=$?"
