# MMA issue probe; ncu of both SpMM kernels on the C3 headline; residual item order A/B (C3/C4/C5)
set -x
timeout 300 tools/probes/probe_mma_issue > gpurun_out/probe_mma_issue.txt 2>&1; echo probe=$?; tail -50 gpurun_out/probe_mma_issue.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
W=c3-reddit-f128-1:2:4
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/r02_launches_c3.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu --no-cusparse --layout natural --no-reorder > gpurun_out/r02_launches_bench.log 2>&1; echo launches=$?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_spmm_full|k_residual" -s 4 -c 2 -o gpurun_out/r02_c3 -f \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-cusparse --layout natural --no-reorder > gpurun_out/r02_ncu_c3.log 2>&1; echo ncu=$?
summ() { python - $1 <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']; pp=d['preprocess']
    print(sys.argv[1], d['config']['workload'], 'tau', d['config']['tau'], d['config']['layout'], 'step %.3f'%d['ms_per_step'], '%.0f GF/s'%d['value'], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()), 'res', pp.get('residual_nnz'))
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
for ord in 0 1; do
  NM_NVCC_FLAGS="-DNM_RES_ORDER=$ord" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/build_$ord.log 2>&1
  for wl in c3-reddit-f128-1:2:4 c4-proteins-f256-128:2:16 c5-products-f100-128:2:8; do
    timeout 900 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl > gpurun_out/ord${ord}_$wl.json 2> gpurun_out/ord${ord}_$wl.err
    summ gpurun_out/ord${ord}_$wl.json
  done
done
