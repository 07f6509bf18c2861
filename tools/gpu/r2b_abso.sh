# same-box A/B of two builds of libgd.so (tools/ab_libs/libgd_{A,B}.so), alternating
set -u
mkdir -p gpurun_out/abso
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
L=paper_conf_icpp_jiangj024_b200/libgd.so
for C in products tiny; do
for V in A B A B A B; do
    cp tools/ab_libs/libgd_$V.so $L
    timeout 900 python bench.py --config $C $A > gpurun_out/abso/${C}_$V.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/abso/${C}_$V.json').readline());print('$C $V',d['value'],d['e2e']['value'],d['roofline']['frac'])"
done
done
for V in A B; do
  cp tools/ab_libs/libgd_$V.so $L
  timeout 900 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum --kernel-name-base function -k regex:'^k_(relabel|sample)_pad' --csv --log-file gpurun_out/abso/warm_$V.csv \
    python bench.py --config products --steps 6 --warmup 3 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e > /dev/null 2>&1; echo ncu $V=$?
  python tools/launch_table.py gpurun_out/abso/warm_$V.csv 2>/dev/null | head -5
done
