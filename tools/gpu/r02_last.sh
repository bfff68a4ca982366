# format 3 with 4 groups A/B; every GPU test; smoke; headline bench
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
summ() { python - $1 <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
    print(sys.argv[1].split('/')[-1], 'tau', d['config']['tau'], 'step %.3f'%d['ms_per_step'], '%.0f GF/s'%d['value'], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()))
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
for wl in c3-reddit-f128-1:2:4 c4-proteins-f256-128:2:16 c2-banded-n1m-d16-f128-1:2:4; do
  for fmt in 1 3; do
    timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl --layout natural --no-reorder --sptc-format $fmt > gpurun_out/l_${fmt}_$wl.json 2> gpurun_out/l_${fmt}_$wl.err
    summ gpurun_out/l_${fmt}_$wl.json
  done
done
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider --durations=10 > gpurun_out/l_gpu_tests.log 2>&1; echo tests=$?; tail -15 gpurun_out/l_gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/l_smoke.log 2>&1; echo smoke=$?; tail -3 gpurun_out/l_smoke.log
timeout 1200 python bench.py > gpurun_out/l_bench_c3.json 2> gpurun_out/l_bench_c3.err; echo bench=$?; tail -c 300 gpurun_out/l_bench_c3.json
