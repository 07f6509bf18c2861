set -u
python tools/build_native.py > /dev/null
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
for r in 1 2 3; do
for KT in 1 0; do
GD_KERNEL_TIMING=$KT timeout 900 python bench.py $A > gpurun_out/kt.json 2> gpurun_out/kt.err; python -c "
import json;d=json.loads(open('gpurun_out/kt.json').read().splitlines()[-1]);print('kt=$KT', d['value'], d['e2e']['value'])"
done
done
