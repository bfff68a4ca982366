# nm_pack_auto (tau by the time model), host Stage-2 tables, C3 full-reorder experiment, filtered launch list
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_score_patterns.py tests/test_parity_reorder_gpu.py tests/test_abi.py -q --timeout 600 -p no:cacheprovider > gpurun_out/t_auto.log 2>&1; echo tests=$?; tail -5 gpurun_out/t_auto.log
summ() { python - $1 <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']; pp=d['preprocess']
    print(sys.argv[1].split('/')[-1], 'tau', d['config']['tau'], d['config']['layout'], 'step %.3f'%d['ms_per_step'], '%.0f GF/s'%d['value'], ' '.join('%s %.3f (%s %.2f)'%(n,v['ms'],v['bound'],v['frac']) for n,v in k.items()), 'reorder_s %.1f'%pp.get('reorder_s',0))
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
for wl in c3-reddit-f128-1:2:4 c2-banded-n1m-d16-f128-1:2:4 c2-banded-n262k-d16-f128-64:2:8 c5-products-f100-128:2:8 c4-proteins-f256-128:2:16; do
  timeout 900 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl > gpurun_out/auto_$wl.json 2> gpurun_out/auto_$wl.err
  summ gpurun_out/auto_$wl.json
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_spmm|k_residual|k_permute" -c 200 --csv --log-file gpurun_out/r02_launches_c3.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-cusparse > gpurun_out/launches_bench.log 2>&1; echo launches=$?
timeout 1500 python tools/c3_reorder_exp.py gpurun_out/c3_reorder_exp.jsonl > gpurun_out/c3_reorder_exp.log 2>&1; echo c3exp=$?; cat gpurun_out/c3_reorder_exp.jsonl
