# record prefetch distance x record evict-first fraction (k_spmm_full)
set -x
for cfg in "0 1.0" "4 1.0" "8 1.0" "12 1.0"; do
  set -- $cfg
  NM_NVCC_FLAGS="-DNM_FULL_PF=$1 -DNM_FULL_REC_FRAC=$2" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/build_pf.log 2>&1 || { echo buildfail; tail -3 gpurun_out/build_pf.log; }
  for wl in c3-reddit-f128-1:2:4 c4-proteins-f256-128:2:16 c2-banded-n1m-d16-f128-1:2:4; do
    timeout 600 python bench.py --no-cpu --no-cusparse --steps 30 --workload $wl --layout natural --no-reorder --sptc-format 1 > gpurun_out/pf_$1_$2_$wl.json 2> /dev/null
    python -c "
import json; d=json.loads(open('gpurun_out/pf_$1_$2_$wl.json').read().strip().splitlines()[-1]); print('pf $1 $2 $wl', '%.3f'%d['ms_per_step'], {k:round(v['ms'],3) for k,v in d['roofline']['kernels'].items()})"
  done
done
