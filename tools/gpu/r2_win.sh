set -u
python tools/build_native.py > /dev/null
for r in 1 2 3 4; do
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 --window 4 --no-cpu-baseline > gpurun_out/w$r.json 2> gpurun_out/w$r.err; python -c "
import json;d=json.loads(open('gpurun_out/w$r.json').read().splitlines()[-1]);print($r, d['value'], d['windows'], d['e2e']['value'], d['e2e']['windows'])"
done
