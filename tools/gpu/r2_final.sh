# round-2 final evidence on one box: smoke, GPU tests, every config's default bench line (+ the
# driver's 20-step papers100m command), f4 train lines, compute-sanitizer on the new code paths
set -u
mkdir -p gpurun_out/final
python tools/build_native.py > /dev/null
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/final/smoke.log 2>&1; echo smoke=$?
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/final/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 gpurun_out/final/pytest_gpu.log
for C in papers100m products friendster mag240m tiny; do
  timeout 1500 python bench.py --config $C --out gpurun_out/final/r02_${C}_bench.json > gpurun_out/final/r02_${C}_bench.log 2>&1; echo "$C rc=$?"
done
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 --out gpurun_out/final/r02_papers100m_driver_cmd.json > gpurun_out/final/drv.log 2>&1; echo drv=$?
timeout 900 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/final/r02_reference.json 2> gpurun_out/final/ref.log; echo ref=$?
for C in products papers100m; do
  timeout 900 python bench.py --config $C --train --steps 100 --no-cpu-baseline --parity-batches 0 --no-replay \
      --out gpurun_out/final/r02_${C}_train.json > gpurun_out/final/r02_${C}_train.log 2>&1; echo "$C train rc=$?"
done
for T in memcheck racecheck synccheck; do
  GD_HOST_THREADS=2 timeout 1200 compute-sanitizer --tool $T --kernel-name regex=k_ python -m pytest tests/test_gpu_parity.py -m gpu -q \
      -k "gather_variants and 512 or tiny_evict or figure6" > gpurun_out/final/san_$T.log 2>&1; echo "san $T rc=$?"; tail -3 gpurun_out/final/san_$T.log
done
A="--steps 100 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e"
for C in papers100m products mag240m; do
  timeout 900 python bench.py --config $C $A --timeline gpurun_out/final/r02_${C}_timeline.md > /dev/null 2>&1; echo "timeline $C rc=$?"
done
