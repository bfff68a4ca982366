# build, every GPU test (no -x: full report), smoke, tau sweep, sanitizers, headline ncu + launch list
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 3600 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider > gpurun_out/gpu_tests.log 2>&1; echo tests=$?; tail -25 gpurun_out/gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?; tail -2 gpurun_out/smoke.log
run() { timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --no-reorder --workload $1 $3 > gpurun_out/$2.json 2>gpurun_out/$2.err
  python - gpurun_out/$2.json "$2" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
    print(sys.argv[2], d['config']['workload'], 'tau', d['config']['tau'], 'step %.3f'%d['ms_per_step'], '%.0f GF/s'%d['value'], ' '.join('%s %.3f (%s %.2f)'%(n,v['ms'],v['bound'],v['frac']) for n,v in k.items()), 'res', d['preprocess']['residual_nnz'])
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
for wl in c3-reddit-f128-1:2:4 c3-reddit-f128-128:2:16 c4-proteins-f256-128:2:16 c5-products-f100-128:2:8; do
  for tau in 2 4 6 8 12; do run $wl tau_${wl}_$tau "--tau $tau"; done
done
for tool in racecheck synccheck memcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_spmm.py > gpurun_out/sanitize_$tool.log 2>&1; echo $tool rc=$?; tail -3 gpurun_out/sanitize_$tool.log
done
