set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_parity_pack_spmm.py -q --timeout 600 -k "fused or hub or formats or concurrent" > gpurun_out/t_fused2.log 2>&1; echo tests=$?; tail -5 gpurun_out/t_fused2.log
run() { timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --no-reorder --workload $1 $3 > gpurun_out/$2.json 2>gpurun_out/$2.err
  python - gpurun_out/$2.json "$2" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
    print(sys.argv[2], d['config']['workload'], 'step %.3f'%d['ms_per_step'], '%.0f GF/s'%d['value'], ' '.join('%s %.3f (%s %.2f)'%(n,v['ms'],v['bound'],v['frac']) for n,v in k.items()))
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
run c3-reddit-f128-1:2:4 f2_c3
run c4-proteins-f256-128:2:16 f2_c4
run c5-products-f100-128:2:8 f2_c5
run c2-banded-n1m-d16-f128-1:2:4 f2_c2
