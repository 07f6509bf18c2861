# final refresh after k_relabel_pad went to 4 positions per thread: GPU tests, smoke, every config's
# default line, the driver's command, the reference arm, train lines, warm launch lists, timelines
set -u
O=gpurun_out/final6
mkdir -p $O
python tools/build_native.py > /dev/null
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?; tail -1 $O/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > $O/pytest_gpu.log 2>&1; echo pytest=$?; tail -2 $O/pytest_gpu.log
for C in products tiny papers100m friendster mag240m; do
  timeout 1500 python bench.py --config $C --out $O/r02_${C}_bench.json > $O/r02_${C}_bench.log 2>&1; echo "$C rc=$?"
  python -c "import json;d=json.loads(open('$O/r02_${C}_bench.json').readline());print(' ',d['value'],d['e2e']['value'],d['roofline']['frac'],d.get('roofline_gather',d['roofline'])['frac'],d['parity']['bit_exact'],(d['roofline'].get('per_path_GBps') or {}).get('host_gather_phase1'))"
done
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 --out $O/r02_papers100m_driver_cmd.json > $O/drv.log 2>&1; echo drv=$?
timeout 900 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > $O/r02_reference.json 2> $O/ref.log; echo ref=$?
for C in products papers100m; do
  timeout 900 python bench.py --config $C --train --steps 100 --no-cpu-baseline --parity-batches 0 --no-replay \
      --out $O/r02_${C}_train.json > $O/r02_${C}_train.log 2>&1; echo "$C train rc=$?"
done
A="--steps 100 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e"
for C in products papers100m mag240m; do
  timeout 900 python bench.py --config $C $A --timeline $O/r02_${C}_timeline.md > /dev/null 2>&1; echo "timeline $C rc=$?"
done
for C in products papers100m; do
  timeout 900 ncu --cache-control none --clock-control none --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum \
    --kernel-name-base function -k regex:'^k_' --csv --log-file $O/${C}_warm.csv \
    python bench.py --config $C --steps 6 --warmup 3 --no-cpu-baseline --parity-batches 0 --no-replay --no-e2e > /dev/null 2>&1; echo "warm $C rc=$?"
done
SKIP=8 OUT=$O bash tools/profile.sh products k_relabel_pad > /dev/null 2>&1; echo "full rc=$?"
