set -u
python tools/build_native.py > /dev/null
timeout 900 python -m pytest tests/test_gpu_bench.py -q -x > gpurun_out/t_kt2.log 2>&1; echo pytest=$?; tail -1 gpurun_out/t_kt2.log
for r in 1 2; do
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/kt2_$r.json 2> gpurun_out/kt2_$r.err; python -c "
import json;d=json.loads(open('gpurun_out/kt2_$r.json').read().splitlines()[-1]);print('drv', d['value'], d['e2e']['value'], d['roofline']['frac'], d['roofline_gather']['frac'], d['roofline_miss']['per_path_GBps'], d['parity']['bit_exact'])"
done
timeout 900 python bench.py --steps 200 --warmup 16 --no-cpu-baseline > gpurun_out/kt2_200.json 2> gpurun_out/kt2_200.err; python -c "
import json;d=json.loads(open('gpurun_out/kt2_200.json').read().splitlines()[-1]);print('200', d['value'], d['e2e']['value'], d['roofline']['frac'], d['roofline_gather']['frac'], d['per_batch'])"
