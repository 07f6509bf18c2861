#!/bin/bash
# ncu evidence for one config (run under gpurun, 1 GPU):
#   launches_<cfg>.csv : every libgd kernel launch with its device time (cold, serialised)
#   prof_<kernel>_<cfg>.ncu-rep : --set full of the given kernels
# usage: tools/profile.sh <config> [kernel regex ...]
set -u
CFG=${1:-papers100m}; shift || true
OUT=gpurun_out
mkdir -p $OUT
ARGS="--config $CFG --steps 6 --warmup 3 --no-cpu-baseline --no-e2e --parity-batches 0"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --kernel-name-base function \
    -k regex:'^k_' --csv --log-file $OUT/launches_$CFG.csv python bench.py $ARGS > $OUT/ncu_launches_$CFG.log 2>&1
echo "launches rc=$?"
for K in "$@"; do
  timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base function \
      -k regex:"^$K\$" -s 4 -c 2 -o $OUT/prof_${K}_$CFG -f python bench.py $ARGS > $OUT/ncu_${K}_$CFG.log 2>&1
  echo "$K rc=$?"
done
