# full-record vs compressed-record tensor-core kernel: parity tests, then bench A/B on C3 + C2
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_parity_pack_spmm.py -x -q -k "formats or concurrent or residual_split or spmm" > gpurun_out/t_fmt.log 2>&1; echo rc=$?; tail -5 gpurun_out/t_fmt.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?; tail -2 gpurun_out/smoke.log
for wl in c3-reddit-f128-1:2:4 c2-banded-n1m-d16-f128-1:2:4; do
 for fmt in 1 2; do
  timeout 900 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl --max-outer 0 --max-stage1 -1 --max-stage2 -1 --sptc-format $fmt > gpurun_out/ab_${wl}_$fmt.json 2> gpurun_out/ab_${wl}_$fmt.err
  python - gpurun_out/ab_${wl}_$fmt.json <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
    print(sys.argv[1], '%.0f GF/s'%d['value'], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()), 'chunks', d['preprocess']['n_chunks'])
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
 done
done
