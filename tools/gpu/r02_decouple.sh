# sptc gathers decoupled from the record copy: parity tests + bench C2/C3/C4/C5
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/test_parity_pack_spmm.py tests/test_parity_gnn_fullsize.py tests/test_parity_fullsize.py tests/test_parity_models.py -q -x --timeout 900 -p no:cacheprovider -k "not bench_launch" > gpurun_out/t_dec.log 2>&1; echo tests=$?; tail -5 gpurun_out/t_dec.log
summ() { python - $1 <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']; pp=d['preprocess']
    print(sys.argv[1], d['config']['workload'], 'tau', d['config']['tau'], d['config']['layout'], 'step %.3f'%d['ms_per_step'], '%.0f GF/s'%d['value'], ' '.join('%s %.3f (%s %.2f)'%(n,v['ms'],v['bound'],v['frac']) for n,v in k.items()), 'res', pp.get('residual_nnz'))
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
for wl in c3-reddit-f128-1:2:4 c2-banded-n1m-d16-f128-1:2:4 c4-proteins-f256-128:2:16 c3-reddit-f128-128:2:16; do
  timeout 900 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl > gpurun_out/dec_$wl.json 2> gpurun_out/dec_$wl.err
  summ gpurun_out/dec_$wl.json
done
