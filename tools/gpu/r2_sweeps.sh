set -u
python tools/build_native.py > /dev/null
A="--steps 100 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e"
timeout 900 python bench.py --config papers100m $A --timeline gpurun_out/r02_papers100m_timeline.md > gpurun_out/tl_papers.json 2> gpurun_out/tl_papers.err; echo tl_papers=$?
timeout 900 python bench.py --config products $A --timeline gpurun_out/r02_products_timeline.md > gpurun_out/tl_products.json 2> gpurun_out/tl_products.err; echo tl_products=$?
B="--config papers100m --steps 30 --warmup 3 --no-cpu-baseline --no-e2e --parity-batches 0 --no-replay --prewarm-max 64"
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:'^k_gather_rows$' -s 60 -c 1 -o gpurun_out/prof_k_gather_rows_papers100m -f python bench.py $B > gpurun_out/ncu_gr.log 2>&1; echo ncu_gr=$?
GD_GATHER_TMA=1 timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:'^k_gather_tma$' -s 60 -c 1 -o gpurun_out/prof_k_gather_tma_papers100m -f python bench.py $B > gpurun_out/ncu_gt.log 2>&1; echo ncu_gt=$?
timeout 3000 python tools/sweeps.py r02 papers100m 100 > gpurun_out/sweeps.log 2>&1; echo sweeps=$?
cp -r profiles/r02_sweeps profiles/r02_sweeps_papers100m.md gpurun_out/ 2>/dev/null
