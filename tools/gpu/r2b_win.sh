# per-window rates of the timed and e2e regions (mag240m, papers100m); sanitizer on the padded sampler
set -u
mkdir -p gpurun_out/win
python tools/build_native.py > /dev/null
A="--no-cpu-baseline --parity-batches 0 --no-replay --window 50"
for C in mag240m papers100m; do
  for i in 1 2; do
    timeout 900 python bench.py --config $C --steps 600 --warmup 8 $A > gpurun_out/win/${C}_$i.json 2> gpurun_out/win/${C}_$i.log
    python -c "import json;d=json.loads(open('gpurun_out/win/${C}_$i.json').readline());print('$C',d['value'],d['e2e']['value']);print(' timed',d['windows']);print(' e2e',d['e2e']['windows']);print(d['miss_policy'])"
  done
done
for T in memcheck synccheck; do
  timeout 900 compute-sanitizer --tool $T --kernel-name regex=k_ python -m pytest tests/test_gpu_parity.py -m gpu -q -x \
      -k "sample_parity_tiny or multi_tile or edge_cases or tiny_evict" > gpurun_out/win/san_$T.log 2>&1; echo "san $T rc=$?"; tail -3 gpurun_out/win/san_$T.log
done
