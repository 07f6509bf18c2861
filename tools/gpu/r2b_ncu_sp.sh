# --set full of the third-hop k_sample_pad (products), final code
set -u
O=gpurun_out/ncusp2
mkdir -p $O
python tools/build_native.py > /dev/null
ARGS="--steps 6 --warmup 3 --no-cpu-baseline --no-e2e --parity-batches 0 --no-replay --prewarm-max 64"
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base function -k regex:'^k_sample_pad$' -s 8 -c 1 \
   -o $O/prof_k_sample_pad_products -f python bench.py --config products $ARGS > $O/ncu_sp.log 2>&1; echo sp=$?
ls $O
