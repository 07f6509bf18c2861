# refresh of the miss-path lines with the per-config sample-ahead default (0 with a miss path),
# the driver's command and the reference arm (its config must match the GPU arm's), GPU bench tests
set -u
O=gpurun_out/final5
mkdir -p $O
python tools/build_native.py > /dev/null
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
timeout 1200 python -m pytest tests/test_gpu_bench.py -m gpu -q -x > $O/pytest_bench.log 2>&1; echo pytest_bench=$?; tail -1 $O/pytest_bench.log
for C in papers100m friendster mag240m; do
  timeout 1500 python bench.py --config $C --out $O/r02_${C}_bench.json > $O/r02_${C}_bench.log 2>&1; echo "$C rc=$?"
  python -c "import json;d=json.loads(open('$O/r02_${C}_bench.json').readline());print(' ',d['value'],d['e2e']['value'],d['roofline']['frac'],d['roofline_gather']['frac'],d['parity']['bit_exact'],d['roofline']['per_path_GBps']['host_gather_phase1'],d['config']['batches_in_flight'])"
done
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 --out $O/r02_papers100m_driver_cmd.json > $O/drv.log 2>&1; echo drv=$?
timeout 900 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > $O/r02_reference.json 2> $O/ref.log; echo ref=$?
timeout 900 python bench.py --config papers100m --train --steps 100 --no-cpu-baseline --parity-batches 0 --no-replay \
      --out $O/r02_papers100m_train.json > $O/r02_papers100m_train.log 2>&1; echo "papers train rc=$?"
A="--steps 100 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e"
for C in papers100m mag240m; do
  timeout 900 python bench.py --config $C $A --timeline $O/r02_${C}_timeline.md > /dev/null 2>&1; echo "timeline $C rc=$?"
done
