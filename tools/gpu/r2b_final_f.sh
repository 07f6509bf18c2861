# final lines after the e2e region got its own W warm-up steps: bench GPU tests, all five default
# lines, the driver's command, the reference arm
set -u
O=gpurun_out/final7
mkdir -p $O
python tools/build_native.py > /dev/null
timeout 1200 python -m pytest tests/test_gpu_bench.py -m gpu -q -x > $O/pytest_bench.log 2>&1; echo pytest_bench=$?; tail -1 $O/pytest_bench.log
for C in papers100m products friendster mag240m tiny; do
  timeout 1500 python bench.py --config $C --out $O/r02_${C}_bench.json > $O/r02_${C}_bench.log 2>&1; echo "$C rc=$?"
  python -c "import json;d=json.loads(open('$O/r02_${C}_bench.json').readline());print(' ',d['value'],d['e2e']['value'],d['roofline']['frac'],d.get('roofline_gather',d['roofline'])['frac'],d['parity']['bit_exact'],(d['roofline'].get('per_path_GBps') or {}).get('host_gather_phase1'))"
done
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 --out $O/r02_papers100m_driver_cmd.json > $O/drv.log 2>&1; echo drv=$?
python -c "import json;d=json.loads(open('$O/r02_papers100m_driver_cmd.json').readline());print(' ',d['value'],d['e2e']['value'],d['roofline']['frac'])"
timeout 900 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > $O/r02_reference.json 2> $O/ref.log; echo ref=$?
