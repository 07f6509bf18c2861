# round-2 re-entry: validate the checkpointed head on one box (smoke, GPU tests, two bench lines)
set -u
mkdir -p gpurun_out/r2b
python tools/build_native.py > /dev/null
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2b/smoke.log 2>&1; echo smoke=$?
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/r2b/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 gpurun_out/r2b/pytest_gpu.log
for C in papers100m products; do
  timeout 1200 python bench.py --config $C --out gpurun_out/r2b/${C}_bench.json > gpurun_out/r2b/${C}_bench.log 2>&1; echo "$C rc=$?"
  tail -c 600 gpurun_out/r2b/${C}_bench.log
done
