set -u
python tools/build_native.py > /dev/null
for r in 1 2 3 4 5; do
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 --no-cpu-baseline --parity-batches 0 --no-replay > gpurun_out/d6_$r.json 2> gpurun_out/d6_$r.err; echo "drv$r rc=$?"
done
