set -u
python tools/build_native.py > /dev/null
A="--steps 100 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e"
for C in papers100m products mag240m; do
timeout 900 python bench.py --config $C $A --timeline gpurun_out/r02_${C}_timeline.md > gpurun_out/tl_$C.json 2> gpurun_out/tl_$C.err; echo "$C=$?"
done
timeout 1200 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sector_hit_rate.pct --cache-control none --clock-control none --kernel-name-base function \
    -k regex:'^k_' --csv --log-file gpurun_out/launches_warm_products.csv python bench.py --config products --steps 6 --warmup 3 --no-cpu-baseline --no-e2e --parity-batches 0 --no-replay > gpurun_out/ncu_warm.log 2>&1; echo ncu=$?
