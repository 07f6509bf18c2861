set -u
mkdir -p gpurun_out/rp
python tools/build_native.py > /dev/null
ARGS="--config products --steps 6 --warmup 3 --no-cpu-baseline --no-e2e --parity-batches 0 --no-replay"
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base function \
   -k regex:'^k_relabel_pad' -s 30 -c 3 -o gpurun_out/rp/relabel_pad -f python bench.py $ARGS > gpurun_out/rp/ncu.log 2>&1; echo rc=$?
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base function \
   -k regex:'^k_sample_pad' -s 30 -c 3 -o gpurun_out/rp/sample_pad -f python bench.py $ARGS > gpurun_out/rp/ncu2.log 2>&1; echo rc=$?
