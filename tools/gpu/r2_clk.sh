set -u
python tools/build_native.py > /dev/null
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
for r in 1 2 3; do
for P in 0.2 0; do
GD_CLOCK_PERIOD_S=$P timeout 900 python bench.py $A > gpurun_out/ck.json 2> gpurun_out/ck.err; python -c "
import json;d=json.loads(open('gpurun_out/ck.json').read().splitlines()[-1]);print('period=$P', d['value'], d['e2e']['value'], d['roofline_miss']['per_path_GBps']['staged_copy_engine_h2d'], d['clocks']['samples'])"
done
done
