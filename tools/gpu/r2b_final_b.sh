# second box for the host-link-bound configs (the host side varies box to box), plus the
# --set full captures the first pass skipped past (too few launches for -s 20)
set -u
O=gpurun_out/final3
mkdir -p $O
python tools/build_native.py > /dev/null
python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
for C in papers100m friendster mag240m; do
  timeout 1500 python bench.py --config $C --out $O/r02_${C}_bench.json > $O/r02_${C}_bench.log 2>&1; echo "$C rc=$?"
  python -c "import json;d=json.loads(open('$O/r02_${C}_bench.json').readline());print(' ',d['value'],d['e2e']['value'],d['roofline']['frac'],d.get('roofline_gather',d['roofline'])['frac'],d['parity']['bit_exact'],d['roofline']['per_path_GBps']['host_gather_phase1'])"
done
timeout 900 python bench.py --gpus 1 --steps 20 --warmup 5 --out $O/r02_papers100m_driver_cmd.json > $O/drv.log 2>&1; echo drv=$?
SKIP=8 OUT=$O bash tools/profile.sh products 'k_sample_pad<8>' k_lookup k_release 'k_gather_rows.*' > /dev/null 2>&1; echo "full products rc=$?"
SKIP=8 OUT=$O bash tools/profile.sh papers100m k_pop_assign k_relabel_pad > /dev/null 2>&1; echo "full papers rc=$?"
ls $O
