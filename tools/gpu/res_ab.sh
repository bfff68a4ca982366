set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_parity_pack_spmm.py -x -q -k "formats or concurrent or residual_split" > gpurun_out/t_res.log 2>&1; echo rc=$?; tail -3 gpurun_out/t_res.log
for wl in c3-reddit-f128-1:2:4 c5-products-f100-128:2:8; do
  timeout 900 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl --max-outer 0 --max-stage1 -1 --max-stage2 -1 > gpurun_out/r_$wl.json 2> gpurun_out/r_$wl.err
  python - gpurun_out/r_$wl.json <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']; pp=d['preprocess']
    print(sys.argv[1], '%.0f GF/s'%d['value'], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()), 'chunks', pp['n_chunks'], 'res', pp['residual_nnz'], 'items', pp['residual_items'], 'split', pp['residual_split_rows'])
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
done
