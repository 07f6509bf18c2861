#!/bin/bash
# ncu evidence for one config (run under gpurun, 1 GPU):
#   launches_<cfg>.csv : every libgd kernel launch: device time + DRAM/PCIe bytes (one pass each)
#   prof_<kernel>_<cfg>.ncu-rep : --set full of the given kernels (HBM-side kernels; the miss
#                                 copies write GBs of slots, which makes ncu's replay impractical)
# usage: tools/profile.sh <config> [kernel regex ...]
set -u
CFG=${1:-papers100m}; shift || true
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
ARGS="--config $CFG --steps 6 --warmup 3 --no-cpu-baseline --no-e2e --parity-batches 0 --prewarm-max 64"
METRICS=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,pcie__read_bytes.sum,pcie__write_bytes.sum,lts__t_sectors_srcunit_tex_aperture_sysmem.sum
timeout 1200 ncu --metrics $METRICS --clock-control none --kernel-name-base function \
    -k regex:'^k_' --csv --log-file $OUT/launches_$CFG.csv python bench.py $ARGS > $OUT/ncu_launches_$CFG.log 2>&1
echo "launches rc=$?"
for K in "$@"; do
  KN=$(printf '%s' "$K" | tr -c 'A-Za-z0-9_' '_')
  timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base function \
      -k regex:"^$K\$" -s ${SKIP:-8} -c 1 -o $OUT/prof_${KN}_$CFG -f python bench.py $ARGS > $OUT/ncu_${KN}_$CFG.log 2>&1
  echo "$K rc=$?"
done
