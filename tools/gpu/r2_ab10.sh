set -u
python tools/build_native.py > /dev/null
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
for PF in auto 8 2 4; do
for C in mag240m friendster; do
if [ $PF = auto ]; then E=""; else E="GD_GATHER_PF=$PF"; fi
env $E timeout 900 python bench.py --config $C $A > gpurun_out/pf_${PF}_$C.json 2> gpurun_out/pf_${PF}_$C.err; python -c "
import json;d=json.loads(open('gpurun_out/pf_${PF}_$C.json').read().splitlines()[-1]);print('$PF', '$C', d['value'], d['roofline']['frac'], d['roofline_miss']['per_path_GBps'], d['miss_policy']['zero_copy_share'])"
done
done
