set -u
python tools/build_native.py > /dev/null
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
for RG in 4 8 4 8 12; do
for C in papers100m mag240m; do
GD_STAGE_RING=$RG timeout 900 python bench.py --config $C $A > gpurun_out/rg.json 2> gpurun_out/rg.err; python -c "
import json;d=json.loads(open('gpurun_out/rg.json').read().splitlines()[-1]);print('ring=$RG $C', d['value'], d['roofline']['frac'], d['roofline_miss']['per_path_GBps'])"
done
done
