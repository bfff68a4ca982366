set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_parity_pack_spmm.py -x -q -k "formats or concurrent or spmm or hub" > gpurun_out/t_cps.log 2>&1; echo tests=$?; tail -3 gpurun_out/t_cps.log
run() { timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --no-reorder --workload $1 $3 > gpurun_out/$2.json 2>gpurun_out/$2.err
  python - gpurun_out/$2.json "$2" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
    print(sys.argv[2], d['config']['workload'], 'step %.3f'%d['ms_per_step'], ' '.join('%s %.3f (%s %.2f)'%(n,v['ms'],v['bound'],v['frac']) for n,v in k.items()), 'chunks', d['preprocess']['n_chunks'])
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
run c3-reddit-f128-1:2:4 cps_c3
run c3-reddit-f128-1:2:4 cps_c3_cmp "--sptc-format 2"
run c2-banded-n1m-d16-f128-1:2:4 cps_c2
run c4-proteins-f256-128:2:16 cps_c4
run c5-products-f100-128:2:8 cps_c5
NM_NVCC_FLAGS="-DNM_FULL_MMA_ONLY" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/bld_mo.log 2>&1
run c3-reddit-f128-1:2:4 cps_mo_c3
python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/bld_prod.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_spmm_full -s 3 -c 1 -o gpurun_out/r02_c3_full python bench.py --no-cpu --no-cusparse --steps 1 --warmup 3 --no-reorder --workload c3-reddit-f128-1:2:4 > gpurun_out/ncu_a.log 2>&1; echo ncu_a=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_residual -s 3 -c 1 -o gpurun_out/r02_c3_res python bench.py --no-cpu --no-cusparse --steps 1 --warmup 3 --no-reorder --workload c3-reddit-f128-1:2:4 > gpurun_out/ncu_b.log 2>&1; echo ncu_b=$?
ls gpurun_out/*.ncu-rep
