# same-box A/B of the k_sample_pad grid: A = one group per bound node, B = 1184 blocks looping, C = 2368
set -u
mkdir -p gpurun_out/abso4
L=paper_conf_icpp_jiangj024_b200/libgd.so
for V in B C; do
cp tools/ab_libs/libgd_$V.so $L
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -x -k sample > gpurun_out/abso4/pytest_$V.log 2>&1; echo "pytest $V=$?"; tail -1 gpurun_out/abso4/pytest_$V.log
done
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for i in 1 2 3; do
for V in A B C; do
    cp tools/ab_libs/libgd_$V.so $L
    timeout 900 python bench.py --config products $A > gpurun_out/abso4/products_${V}_$i.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/abso4/products_${V}_$i.json').readline());print('products $V',d['value'],d['e2e']['value'])"
done
done
for i in 1 2; do
for V in A B C; do
    cp tools/ab_libs/libgd_$V.so $L
    timeout 900 python bench.py --config papers100m $A > gpurun_out/abso4/papers_${V}_$i.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/abso4/papers_${V}_$i.json').readline());print('papers $V',d['value'],d['e2e']['value'],d['roofline']['frac'])"
done
done
