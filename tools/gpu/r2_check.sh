set -x
python tools/build_native.py >/dev/null
(nproc; lscpu; numactl -H 2>/dev/null; free -g; df -h /dev/shm; nvidia-smi topo -m) > gpurun_out/box.txt 2>&1
python -m pytest tests/test_gpu_bench.py -x -q > gpurun_out/t2.log 2>&1; tail -5 gpurun_out/t2.log
for c in papers100m products tiny; do timeout 600 python bench.py --config $c --steps 20 --warmup 5 > gpurun_out/r2_$c.json 2> gpurun_out/r2_$c.err; tail -c 400 gpurun_out/r2_$c.err; done
