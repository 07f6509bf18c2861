set -u
python tools/build_native.py > /dev/null
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 0 --no-replay"
timeout 900 python bench.py $A > gpurun_out/c_base.json 2> gpurun_out/c_base.err; echo base=$?
GD_STAGE_CHUNK_KB=16384 timeout 900 python bench.py $A > gpurun_out/c_16m.json 2> gpurun_out/c_16m.err; echo 16m=$?
GD_STAGE_CHUNK_KB=4096 timeout 900 python bench.py $A > gpurun_out/c_4m.json 2> gpurun_out/c_4m.err; echo 4m=$?
GD_ZERO_COPY_SHARE=0 timeout 900 python bench.py $A > gpurun_out/c_z0.json 2> gpurun_out/c_z0.err; echo z0=$?
GD_HOST_THREADS=14 timeout 900 python bench.py $A > gpurun_out/c_t14.json 2> gpurun_out/c_t14.err; echo t14=$?
