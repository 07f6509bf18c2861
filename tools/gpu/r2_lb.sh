set -u
python tools/build_native.py > /dev/null
timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/t_lb.log 2>&1; echo pytest=$?; tail -2 gpurun_out/t_lb.log
A="--steps 200 --warmup 16 --no-cpu-baseline --parity-batches 4"
for C in products papers100m tiny; do
timeout 900 python bench.py --config $C $A > gpurun_out/lb_$C.json 2> gpurun_out/lb_$C.err; python -c "
import json;d=json.loads(open('gpurun_out/lb_$C.json').read().splitlines()[-1]);pb=d['per_batch'];print('$C', d['value'], d['e2e']['value'], round(pb['sample_ms_per_batch'],4), round(pb['bookkeeping_ms_per_batch'],4), d['parity']['bit_exact'], d['parity']['steady_state']['batches'])"
done
timeout 1200 ncu --metrics gpu__time_duration.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed --cache-control none --clock-control none --kernel-name-base function \
    -k regex:'^k_' --csv --log-file gpurun_out/launches_warm_products_lb.csv python bench.py --config products --steps 6 --warmup 3 --no-cpu-baseline --no-e2e --parity-batches 0 --no-replay > gpurun_out/ncu_warm_lb.log 2>&1; echo ncu=$?
