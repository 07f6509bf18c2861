#!/bin/bash
# f4 evidence (1 GPU): train parity tests, bench --train, and the ncu launch list of the train step.
#   usage: tools/train_prof.sh [config]
set -u
CFG=${1:-products}
OUT=gpurun_out
mkdir -p $OUT
timeout 600 python -m pytest tests/test_gpu_train.py -x -q > $OUT/pytest_train.log 2>&1; echo "train tests rc=$?"; tail -2 $OUT/pytest_train.log
timeout 600 python bench.py --config $CFG --train --steps 100 --no-cpu-baseline --parity-batches 0 \
    --out $OUT/bench_${CFG}_train.json > $OUT/bench_${CFG}_train.log 2>&1; echo "bench rc=$?"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    --kernel-name-base function -k regex:'^(k_|nvjet|cutlass|sm100|gd_)' --csv --log-file $OUT/launches_${CFG}_train.csv \
    python bench.py --config $CFG --train --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --parity-batches 0 \
    --prewarm-max 8 > $OUT/ncu_train_$CFG.log 2>&1; echo "ncu rc=$?"
