set -u
python tools/build_native.py > /dev/null
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
for C in mag240m papers100m; do
for SH in 0 0.05 adaptive 0; do
if [ $SH = adaptive ]; then E="GD_HOST_THREADS=13"; else E="GD_HOST_THREADS=13 GD_ZERO_COPY_SHARE=$SH"; fi
env $E timeout 900 python bench.py --config $C $A > gpurun_out/zs.json 2> gpurun_out/zs.err; python -c "
import json;d=json.loads(open('gpurun_out/zs.json').read().splitlines()[-1]);pb=d['per_batch'];print('$C $SH', d['value'], d['roofline']['frac'], d['roofline_miss']['per_path_GBps'], round(d['miss_policy']['zero_copy_share'],3), 'zc_rows', d['roofline_miss']['misses_zero_copy']//200)"
done
done
