# A/B on one box: hit-gather variants, THP host table, host-gather threads (papers100m)
python tools/build_native.py >/dev/null
python -m pytest tests/test_gpu_parity.py -q -x -k "gather_variants or adaptive" > gpurun_out/t3.log 2>&1; tail -2 gpurun_out/t3.log
A="--steps 100 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
python bench.py $A > gpurun_out/ab_base.json 2> gpurun_out/ab_base.err
GD_THP=0 python bench.py $A > gpurun_out/ab_nothp.json 2> gpurun_out/ab_nothp.err
GD_GATHER_TMA=1 python bench.py $A > gpurun_out/ab_tma.json 2> gpurun_out/ab_tma.err
GD_GATHER_DYNAMIC=0 GD_GATHER_PRIORITY=0 python bench.py $A > gpurun_out/ab_r1gather.json 2> gpurun_out/ab_r1gather.err
GD_HOST_THREADS=15 python bench.py $A > gpurun_out/ab_t15.json 2> gpurun_out/ab_t15.err
GD_GATHER_TMA=1 python bench.py --config products --steps 100 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay > gpurun_out/ab_prod_tma.json 2> gpurun_out/ab_prod_tma.err
python bench.py --config products --steps 100 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay > gpurun_out/ab_prod.json 2> gpurun_out/ab_prod.err
