set -u
python tools/build_native.py > /dev/null
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
for V in "0 auto" "1 auto" "1 16" "0 16" "1 8"; do
set -- $V
if [ $2 = auto ]; then E="GD_GATHER_PF_HINT=$1"; else E="GD_GATHER_PF_HINT=$1 GD_GATHER_PF=$2"; fi
env $E timeout 900 python bench.py --config papers100m $A > gpurun_out/h.json 2> gpurun_out/h.err; python -c "
import json;d=json.loads(open('gpurun_out/h.json').read().splitlines()[-1]);print('$E', d['value'], d['roofline']['frac'], d['roofline_miss']['per_path_GBps'])"
done
