set -u
python tools/build_native.py > /dev/null
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
for K in 8192 16384 24576 32768 8192 16384 12288; do
GD_STAGE_CHUNK_KB=$K timeout 900 python bench.py $A > gpurun_out/k_$K.json 2> gpurun_out/k_$K.err; echo "$K=$?"; python -c "
import json;d=json.loads(open('gpurun_out/k_$K.json').read().splitlines()[-1]);print($K, d['value'], d['roofline']['frac'], d['roofline_miss']['per_path_GBps'])"
done
for K in 8192 16384; do
GD_STAGE_CHUNK_KB=$K timeout 900 python bench.py --config mag240m $A > gpurun_out/km_$K.json 2> gpurun_out/km_$K.err; python -c "
import json;d=json.loads(open('gpurun_out/km_$K.json').read().splitlines()[-1]);print('mag', $K, d['value'], d['roofline']['frac'], d['roofline_miss']['per_path_GBps'])"
GD_STAGE_CHUNK_KB=$K timeout 900 python bench.py --config friendster $A > gpurun_out/kf_$K.json 2> gpurun_out/kf_$K.err; python -c "
import json;d=json.loads(open('gpurun_out/kf_$K.json').read().splitlines()[-1]);print('fr', $K, d['value'], d['roofline']['frac'], d['roofline_miss']['per_path_GBps'])"
done
