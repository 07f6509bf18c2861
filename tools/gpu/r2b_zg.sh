# zero-copy after the hit gather (A/B): papers100m, mag240m; parity of the ordering
set -u
mkdir -p gpurun_out/zg
python tools/build_native.py > /dev/null
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for C in papers100m mag240m; do
for Z in 0 1 0 1; do
    GD_ZC_AFTER_GATHER=$Z timeout 900 python bench.py --config $C $A > gpurun_out/zg/${C}_$Z.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/zg/${C}_$Z.json').readline());g=d['roofline_gather'];print('$C zg=$Z',d['value'],d['e2e']['value'],'link',d['roofline']['frac'],'gather live',g['frac'],'iso',g['isolated']['frac'],'host',d['roofline']['per_path_GBps']['host_gather_phase1'])"
done
done
GD_ZC_AFTER_GATHER=1 timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "extract or split or release or evict" > gpurun_out/zg/pytest.log 2>&1; echo pytest=$?; tail -2 gpurun_out/zg/pytest.log
