# gather groups walk only their own stages (StageIter): parity + A/B
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/test_parity_pack_spmm.py tests/test_parity_gnn_fullsize.py tests/test_parity_fullsize.py tests/test_parity_gcn.py -q -x --timeout 900 -p no:cacheprovider > gpurun_out/t_addr.log 2>&1; echo tests=$?; tail -4 gpurun_out/t_iter.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_addr.log 2>&1; echo smoke=$?
for wl in c3-reddit-f128-1:2:4 c4-proteins-f256-128:2:16 c2-banded-n1m-d16-f128-1:2:4; do
  for fmt in 1 3; do
    timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl --layout natural --no-reorder --sptc-format $fmt > gpurun_out/ad_${fmt}_$wl.json 2> /dev/null
    python -c "
import json; d=json.loads(open('gpurun_out/ad_${fmt}_$wl.json').read().strip().splitlines()[-1]); print('$wl fmt $fmt', '%.3f'%d['ms_per_step'], {k:round(v['ms'],3) for k,v in d['roofline']['kernels'].items()})"
  done
done
