# same-box A/B/C/D of k_relabel_pad builds (A default: 8 items, 80 regs; B: min 5 blocks/SM, 48 regs + spill;
# C: 4 items per thread; D: min 4 blocks/SM, 64 regs), alternating, products + tiny; parity of the winner is
# covered by the test run on the committed default
set -u
mkdir -p gpurun_out/abso2
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
L=paper_conf_icpp_jiangj024_b200/libgd.so
for C in products; do
for i in 1 2; do
for V in A B C D; do
    cp tools/ab_libs/libgd_$V.so $L
    timeout 900 python bench.py --config $C $A > gpurun_out/abso2/${C}_${V}_$i.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/abso2/${C}_${V}_$i.json').readline());print('$C $V',d['value'],d['e2e']['value'],d['roofline']['frac'])"
done
done
done
for V in A B C D; do
  cp tools/ab_libs/libgd_$V.so $L
  timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k "sample_parity_multi_tile or sample_edge_cases or sample_parity_tiny" > gpurun_out/abso2/pytest_$V.log 2>&1; echo "pytest $V=$?"
  timeout 900 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum --kernel-name-base function -k regex:'^k_relabel_pad' --csv --log-file gpurun_out/abso2/warm_$V.csv \
    python bench.py --config products --steps 6 --warmup 3 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e > /dev/null 2>&1
  python tools/launch_table.py gpurun_out/abso2/warm_$V.csv 2>/dev/null | tail -1
done
