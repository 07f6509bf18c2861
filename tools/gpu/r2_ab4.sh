set -u
python tools/build_native.py > /dev/null
timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "adaptive or miss_paths or peer" > gpurun_out/t4.log 2>&1; echo pytest=$?; tail -2 gpurun_out/t4.log
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0"
for C in papers100m mag240m friendster; do
timeout 900 python bench.py --config $C $A > gpurun_out/tu_on_$C.json 2> gpurun_out/tu_on_$C.err; echo "$C on rc=$?"
GD_SHARE_TUNER=0 timeout 900 python bench.py --config $C $A > gpurun_out/tu_off_$C.json 2> gpurun_out/tu_off_$C.err; echo "$C off rc=$?"
done
timeout 900 python bench.py --config papers100m --steps 20 --warmup 5 > gpurun_out/tu_drv.json 2> gpurun_out/tu_drv.err; echo "drv rc=$?"
