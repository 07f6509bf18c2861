set -u
python tools/build_native.py > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "adaptive or miss_paths or tuner or peer" > gpurun_out/t_ev.log 2>&1; echo pytest=$?; tail -1 gpurun_out/t_ev.log
for r in 1 2 3; do
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 --no-cpu-baseline --parity-batches 0 > gpurun_out/ev_$r.json 2> gpurun_out/ev_$r.err; python -c "
import json;d=json.loads(open('gpurun_out/ev_$r.json').read().splitlines()[-1]);print('drv', d['value'], d['e2e']['value'], d['roofline']['frac'], d['miss_policy']['zero_copy_share'], d['miss_policy']['r_host_GBps'], d['parity']['bit_exact'])"
done
for r in 1 2; do
timeout 900 python bench.py --steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 > gpurun_out/ev200_$r.json 2> gpurun_out/ev200_$r.err; python -c "
import json;d=json.loads(open('gpurun_out/ev200_$r.json').read().splitlines()[-1]);print('200', d['value'], d['e2e']['value'], d['roofline']['frac'], d['miss_policy']['zero_copy_share'], d['parity']['bit_exact'])"
done
