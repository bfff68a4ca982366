set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_parity_pack_spmm.py -x -q -k "formats or concurrent or spmm or hub" > gpurun_out/t_l2.log 2>&1; echo tests=$?; tail -2 gpurun_out/t_l2.log
run() { timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --no-reorder --workload $1 $3 > gpurun_out/$2.json 2>gpurun_out/$2.err
  python - gpurun_out/$2.json "$2" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
    print(sys.argv[2], d['config']['workload'], 'step %.3f'%d['ms_per_step'], ' '.join('%s %.3f (%s %.2f)'%(n,v['ms'],v['bound'],v['frac']) for n,v in k.items()), 'chunks', d['preprocess']['n_chunks'])
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
run c3-reddit-f128-1:2:4 l2_c3
run c3-reddit-f128-128:2:16 l2_c3b
run c2-banded-n1m-d16-f128-1:2:4 l2_c2
run c4-proteins-f256-128:2:16 l2_c4
run c5-products-f100-128:2:8 l2_c5
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_spmm_full|k_residual" -s 6 -c 2 -o gpurun_out/r02_c3_l2pol python bench.py --no-cpu --no-cusparse --steps 1 --warmup 3 --no-reorder --workload c3-reddit-f128-1:2:4 > gpurun_out/ncu_c.log 2>&1; echo ncu=$?
