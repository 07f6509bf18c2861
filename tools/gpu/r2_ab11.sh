set -u
python tools/build_native.py > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "miss_paths or release_on or adaptive or tiny" > gpurun_out/t11.log 2>&1; echo pytest=$?; tail -1 gpurun_out/t11.log
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
for C in papers100m mag240m friendster; do
for SP in 4000 0; do
GD_POOL_SPIN=$SP timeout 900 python bench.py --config $C $A > gpurun_out/sp_${SP}_$C.json 2> gpurun_out/sp_${SP}_$C.err; python -c "
import json;d=json.loads(open('gpurun_out/sp_${SP}_$C.json').read().splitlines()[-1]);print('$C spin=$SP', d['value'], d['roofline']['frac'], d['roofline_miss']['per_path_GBps'], round(d['miss_policy']['zero_copy_share'],3))"
done
done
for CF in 0 1; do
GD_HASH_CAS_FIRST=$CF timeout 900 python bench.py --config products $A > gpurun_out/cf_$CF.json 2> gpurun_out/cf_$CF.err; python -c "
import json;d=json.loads(open('gpurun_out/cf_$CF.json').read().splitlines()[-1]);print('products cas_first=$CF', d['value'], d['e2e']['value'], round(d['per_batch']['sample_ms_per_batch'],4))"
done
