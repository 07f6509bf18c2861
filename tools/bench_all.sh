#!/bin/bash
# Every config's bench line on one box (DESIGN.md §8 table), then the f4 train runs.
set -u
mkdir -p gpurun_out
for C in papers100m products friendster mag240m tiny; do
  timeout 900 python bench.py --config $C --no-cpu-baseline --out gpurun_out/all_$C.json > gpurun_out/all_$C.log 2>&1; echo "$C rc=$?"
done
for C in papers100m products; do
  timeout 900 python bench.py --config $C --train --steps 100 --no-cpu-baseline --parity-batches 0 \
      --out gpurun_out/all_${C}_train.json > gpurun_out/all_${C}_train.log 2>&1; echo "$C train rc=$?"
done
