set -u
python tools/build_native.py > /dev/null
A="--steps 100 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e"
for S in 1 2; do
  timeout 900 python bench.py --config papers100m --buffer-frac 0.04 $A --samplers $S --timeline gpurun_out/tl_b004_s$S.md > gpurun_out/b004_s$S.json 2> gpurun_out/b004_s$S.err; echo "b004 S=$S rc=$?"
done
timeout 900 python bench.py --config mag240m $A --timeline gpurun_out/tl_mag.md --miss-sweep "13:0.05:0:0,13:0.1:0:0,13:0.2:0:0,13:0.3:0:0,13:0.4:0:0" > gpurun_out/mag_sweep.json 2> gpurun_out/mag_sweep.err; echo mag=$?
timeout 900 python bench.py --config papers100m $A --miss-sweep "13:0.0:0:0,13:0.05:0:0,13:0.1:0:0,13:0.15:0:0,13:0.2:0:0,13:0.3:0:0" > gpurun_out/pap_sweep.json 2> gpurun_out/pap_sweep.err; echo pap=$?
