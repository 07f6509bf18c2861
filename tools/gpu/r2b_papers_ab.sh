# same-box A/B on papers100m (alternating): default | zero-copy share fixed at 0 | --sample-ahead 0
set -u
mkdir -p gpurun_out/pab
python tools/build_native.py > /dev/null
A="--config papers100m --steps 400 --warmup 8 --no-cpu-baseline --parity-batches 0 --no-replay"
for i in 1 2; do
for V in def zc0 ra0 zc0ra0; do
  case $V in
    def) E=""; X="";;
    zc0) E="GD_ZERO_COPY_SHARE=0"; X="";;
    ra0) E=""; X="--sample-ahead 0";;
    zc0ra0) E="GD_ZERO_COPY_SHARE=0"; X="--sample-ahead 0";;
  esac
  env $E timeout 900 python bench.py $A $X > gpurun_out/pab/${V}_$i.json 2>/dev/null
  python -c "import json;d=json.loads(open('gpurun_out/pab/${V}_$i.json').readline());r=d['roofline'];print('$V',d['value'],d['e2e']['value'],'link',r['frac'],'gather',d['roofline_gather']['frac'],'host',r['per_path_GBps']['host_gather_phase1'],'zc',d['miss_policy']['zero_copy_share'])"
done
done
