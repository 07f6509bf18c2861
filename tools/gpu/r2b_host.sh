# host-loop busy time per step vs device time per step (is the host loop the bound?)
set -u
mkdir -p gpurun_out/host
python tools/build_native.py > /dev/null
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for C in tiny products papers100m; do
    timeout 900 python bench.py --config $C $A > gpurun_out/host/$C.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/host/$C.json').readline());print('$C',d['value'],d['ms_per_step'],d['host_loop'])"
done
GD_PDL=0 timeout 900 python bench.py --config products $A > gpurun_out/host/products_nopdl.json 2>/dev/null
python -c "import json;d=json.loads(open('gpurun_out/host/products_nopdl.json').readline());print('products nopdl',d['value'],d['ms_per_step'],d['host_loop'])"
