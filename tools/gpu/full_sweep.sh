# full-record kernel: gather-group count x stage-count sweep on C3 (identity order) + banded C2
set -x
for v in "2 16" "1 16" "4 16" "2 8" "2 12"; do
  set -- $v
  NM_NVCC_FLAGS="-DNM_FULL_GROUPS=$1 -DNM_FULL_MAX_STAGES=$2" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/bld_$1_$2.log 2>&1
  for wl in c3-reddit-f128-1:2:4 c2-banded-n1m-d16-f128-1:2:4; do
    timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl --max-outer 0 --max-stage1 -1 --max-stage2 -1 > gpurun_out/sw_$1_$2_$wl.json 2>/dev/null
    python - gpurun_out/sw_$1_$2_$wl.json "G=$1 S=$2" <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
    print(sys.argv[2], d['config']['workload'], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()))
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
  done
done
