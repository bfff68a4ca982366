# warp-per-item residual kernel: parity tests, then A/B against the subgroup kernel on C2-C5
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/test_parity_pack_spmm.py tests/test_parity_gnn_fullsize.py tests/test_parity_fullsize.py -q -x --timeout 900 -p no:cacheprovider -k "not bench_launch" > gpurun_out/t_resw.log 2>&1; echo tests=$?; tail -15 gpurun_out/t_resw.log
summ() { python - $1 <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']; pp=d['preprocess']
    print(sys.argv[1], d['config']['workload'], 'tau', d['config']['tau'], d['config']['layout'], 'step %.3f'%d['ms_per_step'], '%.0f GF/s'%d['value'], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()), 'res', pp.get('residual_nnz'))
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
for kern in 1 0; do
  NM_NVCC_FLAGS="-DNM_RES_KERNEL=$kern" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/build_$kern.log 2>&1
  for wl in c3-reddit-f128-1:2:4 c4-proteins-f256-128:2:16 c5-products-f100-128:2:8 c2-banded-n1m-d16-f128-1:2:4; do
    timeout 900 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl > gpurun_out/k${kern}_$wl.json 2> gpurun_out/k${kern}_$wl.err
    summ gpurun_out/k${kern}_$wl.json
  done
done
