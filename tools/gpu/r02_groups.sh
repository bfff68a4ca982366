# k_spmm_full gather groups x pipeline depth A/B (compile-time macros), C3 and banded C2
set -x
summ() { python - $1 <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
    print(sys.argv[1].split('/')[-1], 'tau', d['config']['tau'], 'step %.3f'%d['ms_per_step'], '%.0f GF/s'%d['value'], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()))
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
for cfg in "2 16" "4 16"; do
  set -- $cfg
  NM_NVCC_FLAGS="-DNM_FULL_GROUPS=$1 -DNM_FULL_MAX_STAGES=$2" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/build_g$1_$2.log 2>&1 || { echo build-fail $cfg; tail -5 gpurun_out/build_g$1_$2.log; continue; }
  timeout 300 python -m pytest tests/test_parity_pack_spmm.py -q -x -k "formats_agree and (c1 or band)" -p no:cacheprovider > gpurun_out/t_g$1_$2.log 2>&1; echo t=$?
  for wl in c3-reddit-f128-1:2:4 c2-banded-n1m-d16-f128-1:2:4 c4-proteins-f256-128:2:16; do
    timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl --layout natural --no-reorder > gpurun_out/g$1_$2_$wl.json 2> gpurun_out/g$1_$2_$wl.err
    summ gpurun_out/g$1_$2_$wl.json
  done
done
