# confirmation of the committed code: smoke, all GPU tests, the driver's default command
set -u
O=gpurun_out/confirm
mkdir -p $O
python tools/build_native.py > /dev/null
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?; tail -1 $O/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 $O/pytest_gpu.log
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 > $O/drv.json 2> $O/drv.log; echo drv=$?
python -c "import json;d=json.loads(open('$O/drv.json').readline());print(d['value'],d['e2e']['value'],d['roofline']['frac'],d['parity']['bit_exact'],d['gpu_launches'])"
timeout 900 python bench.py > $O/default.json 2> $O/default.log; echo default=$?
python -c "import json;d=json.loads(open('$O/default.json').readline());print(d['value'],d['e2e']['value'],d['roofline']['frac'],d['roofline_gather']['frac'],d['parity']['bit_exact'])"
