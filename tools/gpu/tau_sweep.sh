# hybrid-split threshold sweep (C3 natural + reordered layouts, C4, C5) + compute-sanitizer logs
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for wl in c3-reddit-f128-1:2:4 c4-proteins-f256-128:2:16 c5-products-f100-128:2:8; do
 for tau in 4 6 8 12; do
  timeout 900 python bench.py --no-cpu --no-cusparse --steps 10 --layout natural --tau $tau --workload $wl > gpurun_out/tau_${wl}_$tau.json 2>/dev/null
  python - gpurun_out/tau_${wl}_$tau.json "tau=$tau" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
    print(sys.argv[2], d['config']['workload'], 'step %.3f'%d['ms_per_step'], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()), 'chunks', d['preprocess']['n_chunks'], 'res', d['preprocess']['residual_nnz'])
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
 done
done
for tool in racecheck synccheck memcheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_spmm.py > gpurun_out/sanitize_$tool.log 2>&1; echo $tool rc=$?; tail -3 gpurun_out/sanitize_$tool.log
done
