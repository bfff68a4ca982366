# build, GPU tests, then short bench lines for the given workloads (quick A/B on one box)
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q ${NM_TESTS:-} > gpurun_out/gpu_tests.log 2>&1; echo tests_rc=$?
tail -3 gpurun_out/gpu_tests.log
for wl in ${WLS:-c2-banded-n1m-d16-f128-1:2:4}; do
  for fuse in ${FUSES:-default}; do
    if [ "$fuse" = default ]; then unset NM_RES_FUSE; else export NM_RES_FUSE=$fuse; fi
    timeout 600 python bench.py --no-cpu --no-cusparse --steps 30 --workload $wl 2>&1 | tail -1 > gpurun_out/cb_${wl}_$fuse.json
    python - gpurun_out/cb_${wl}_$fuse.json <<'PY'
import json,sys
try:
    d=json.load(open(sys.argv[1])); k=d['roofline']['kernels']; pp=d['preprocess']
    print('%-60s %7.0f GF/s step %.3f ms '%(sys.argv[1],d['value'],d['ms_per_step'])+'  '.join('%s %.3fms/%.2f'%(n,v['ms'],v['frac']) for n,v in k.items()), 'chunks',pp['n_chunks'],'res',pp['residual_nnz'],'fused',pp.get('residual_nnz_fused'))
except Exception as e: print(sys.argv[1], 'FAILED', e)
PY
  done
done
unset NM_RES_FUSE
