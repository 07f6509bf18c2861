set -u
python tools/build_native.py > /dev/null
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu2.log 2>&1; echo pytest=$?; tail -3 gpurun_out/pytest_gpu2.log
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
for C in products papers100m; do
  for S in 1 2 3; do
    timeout 900 python bench.py --config $C $A --samplers $S > gpurun_out/s${S}_$C.json 2> gpurun_out/s${S}_$C.err; echo "$C S=$S rc=$?"
  done
done
timeout 600 python bench.py --config tiny $A --samplers 2 > gpurun_out/s2_tiny.json 2> gpurun_out/s2_tiny.err
