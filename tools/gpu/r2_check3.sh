set -u
python tools/build_native.py > /dev/null
timeout 900 python -m pytest tests/test_gpu_bench.py -q -x > gpurun_out/pytest_gpu3.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu3.log
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0"
for C in products papers100m; do
  for S in 1 2 3; do
    timeout 900 python bench.py --config $C $A --samplers $S > gpurun_out/s${S}_$C.json 2> gpurun_out/s${S}_$C.err; echo "$C S=$S rc=$?"
  done
done
timeout 600 python bench.py --config tiny $A --samplers 2 > gpurun_out/s2_tiny.json 2> gpurun_out/s2_tiny.err
timeout 600 python bench.py --config tiny $A --samplers 1 > gpurun_out/s1_tiny.json 2> gpurun_out/s1_tiny.err
