set -x
run() { timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --no-reorder --workload $1 > gpurun_out/$2.json 2>gpurun_out/$2.err
  python - gpurun_out/$2.json "$2" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
    print(sys.argv[2], d['config']['workload'], 'step %.3f'%d['ms_per_step'], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()))
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
for v in "base:-DNM_REC_EVICT_FIRST=0 -DNM_X_EVICT_LAST=0" "rec:-DNM_REC_EVICT_FIRST=1 -DNM_X_EVICT_LAST=0" "recx:-DNM_REC_EVICT_FIRST=1 -DNM_X_EVICT_LAST=1" "recx_resx:-DNM_REC_EVICT_FIRST=1 -DNM_X_EVICT_LAST=1 -DNM_RES_X_EVICT_LAST=1" "recx_ldcs:-DNM_REC_EVICT_FIRST=1 -DNM_X_EVICT_LAST=1 -DNM_RES_LDCS=1"; do
  tag=${v%%:*}; flags=${v#*:}
  NM_NVCC_FLAGS="$flags" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/bld_$tag.log 2>&1
  run c3-reddit-f128-1:2:4 pol_${tag}_c3
  run c4-proteins-f256-128:2:16 pol_${tag}_c4
done
