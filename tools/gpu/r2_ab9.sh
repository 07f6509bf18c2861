set -u
python tools/build_native.py > /dev/null
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "miss_paths or release_on or adaptive" > gpurun_out/t9.log 2>&1; echo pytest=$?; tail -1 gpurun_out/t9.log
for C in papers100m mag240m friendster papers100m; do
timeout 900 python bench.py --config $C $A > gpurun_out/a9_$C.json 2> gpurun_out/a9_$C.err; python -c "
import json;d=json.loads(open('gpurun_out/a9_$C.json').read().splitlines()[-1]);print('$C', d['value'], d['roofline']['frac'], d['roofline_miss']['per_path_GBps'], d['parity']['steady_state']['bit_exact'])"
done
