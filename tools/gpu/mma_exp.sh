# MMA-rate experiments inside k_spmm_full (timing-only variants) + ncu of the product kernels on C3
set -x
run() { timeout 900 python bench.py --no-cpu --no-cusparse --steps 10 --layout natural --workload $1 > gpurun_out/$2.json 2>gpurun_out/$2.err
  python - gpurun_out/$2.json "$2" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
    print(sys.argv[2], d['config']['workload'], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()), 'chunks', d['preprocess']['n_chunks'])
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
for v in "MMA_ONLY:-DNM_FULL_MMA_ONLY" "MMA_ALT:-DNM_FULL_MMA_ONLY -DNM_FULL_ALT_ACC" "PROD:"; do
  tag=${v%%:*}; flags=${v#*:}
  NM_NVCC_FLAGS="$flags" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/bld_$tag.log 2>&1
  run c3-reddit-f128-1:2:4 ${tag}_c3
  run c4-proteins-f256-128:2:16 ${tag}_c4
done
WL=c3-reddit-f128-1:2:4
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_full -s 3 -c 1 -o gpurun_out/r02_c3_full python bench.py --no-cpu --no-cusparse --steps 1 --warmup 3 --layout natural --workload $WL > gpurun_out/ncu_a.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_residual -s 3 -c 1 -o gpurun_out/r02_c3_res python bench.py --no-cpu --no-cusparse --steps 1 --warmup 3 --layout natural --workload $WL > gpurun_out/ncu_b.log 2>&1
ls gpurun_out/*.ncu-rep
