set -u
python tools/build_native.py > /dev/null
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "sample or pipeline or run_twice" > gpurun_out/t_cr.log 2>&1; echo pytest=$?; tail -1 gpurun_out/t_cr.log
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 4"
for r in 1 2; do
timeout 900 python bench.py --config products $A > gpurun_out/cr.json 2> gpurun_out/cr.err; python -c "
import json;d=json.loads(open('gpurun_out/cr.json').read().splitlines()[-1]);pb=d['per_batch'];print('products', d['value'], d['e2e']['value'], round(pb['sample_ms_per_batch'],4), d['parity']['bit_exact'])"
done
timeout 1200 ncu --metrics gpu__time_duration.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed --cache-control none --clock-control none --kernel-name-base function \
    -k regex:'^k_col_resolve$' --csv --log-file gpurun_out/cr_ncu.csv python bench.py --config products --steps 6 --warmup 3 --no-cpu-baseline --no-e2e --parity-batches 0 --no-replay > gpurun_out/ncu_cr.log 2>&1; echo ncu=$?
