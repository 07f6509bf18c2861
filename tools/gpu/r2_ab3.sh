set -u
python tools/build_native.py > /dev/null
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
for r in 1 2; do
timeout 900 python bench.py --config papers100m $A > gpurun_out/p_def$r.json 2> gpurun_out/p_def$r.err; echo "def$r rc=$?"
done
timeout 900 python bench.py --config papers100m $A --samplers 1 > gpurun_out/p_s1.json 2> gpurun_out/p_s1.err; echo "s1 rc=$?"
timeout 900 python bench.py --config papers100m $A --no-e2e --miss-sweep "13:0.1:0:0,13:0.15:0:0,13:0.2:0:0,13:0.15:0:0,13:0.1:0:0" > gpurun_out/p_sw.json 2> gpurun_out/p_sw.err; echo "sw rc=$?"
timeout 900 python bench.py --config mag240m $A > gpurun_out/m_def.json 2> gpurun_out/m_def.err; echo "mag rc=$?"
