# round-2 evidence on one box: GPU tests, smoke, every config's default bench line, ncu launch lists
set -u
mkdir -p gpurun_out
python tools/build_native.py > /dev/null
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/pytest_gpu.log
for C in papers100m products friendster mag240m tiny; do
  timeout 1200 python bench.py --config $C --out gpurun_out/r02_${C}_bench.json > gpurun_out/r02_${C}_bench.log 2>&1; echo "$C rc=$?"
done
for C in friendster mag240m papers100m; do
  bash tools/profile.sh $C
done
