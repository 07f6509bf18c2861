# same-box A/B: A = committed k_sample_pad (one group per bound node, no loop), B = 1184 blocks looping
set -u
mkdir -p gpurun_out/abso5
L=paper_conf_icpp_jiangj024_b200/libgd.so
A="--steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for i in 1 2 3; do
for V in A B; do
    cp tools/ab_libs/libgd_$V.so $L
    timeout 900 python bench.py --config products $A > gpurun_out/abso5/products_${V}_$i.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/abso5/products_${V}_$i.json').readline());print('products $V',d['value'],d['e2e']['value'])"
done
done
for V in A B; do
    cp tools/ab_libs/libgd_$V.so $L
    timeout 900 python bench.py --config tiny $A > gpurun_out/abso5/tiny_${V}.json 2>/dev/null
    python -c "import json;d=json.loads(open('gpurun_out/abso5/tiny_${V}.json').readline());print('tiny $V',d['value'],d['e2e']['value'])"
done
