# every GPU test + smoke on the final code
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider --durations=10 > gpurun_out/v_gpu_tests.log 2>&1; echo tests=$?; tail -15 gpurun_out/v_gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/v_smoke.log 2>&1; echo smoke=$?; tail -3 gpurun_out/v_smoke.log
for wl in c2-banded-n1m-d16-f128-1:2:4; do
  for fmt in 1 3; do
    timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl --sptc-format $fmt > gpurun_out/v_${fmt}_$wl.json 2> /dev/null
    python -c "
import json; d=json.loads(open('gpurun_out/v_${fmt}_$wl.json').read().strip().splitlines()[-1]); print('fmt $fmt', d['ms_per_step'], {k:v['ms'] for k,v in d['roofline']['kernels'].items()})"
  done
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_spmm_tm" -s 2 -c 1 -o gpurun_out/r02_c3_tm -f \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-cusparse --layout natural --no-reorder --sptc-format 3 > gpurun_out/ncu_tm.log 2>&1; echo ncu=$?
