# k_residual occupancy variants (batch size x min blocks per SM)
set -x
for cfg in "0 0" "8 3" "4 4" "4 5" "8 1"; do
  set -- $cfg
  if [ "$1" = "0" ]; then F=""; else F="-DNM_RES_BATCH=$1 -DNM_RES_MINB=$2"; fi
  NM_NVCC_FLAGS="$F" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/build_occ.log 2>&1
  timeout 300 python -m pytest tests/test_parity_pack_spmm.py -q -x -k "residual or hybrid" -p no:cacheprovider > gpurun_out/t_occ_$1_$2.log 2>&1; echo t=$?
  for wl in c3-reddit-f128-1:2:4 c4-proteins-f256-128:2:16 c5-products-f100-128:2:8 c2-powerlaw-n262k-d16-f128-1:2:4; do
    timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl --layout natural --no-reorder --sptc-format 1 > gpurun_out/o_$1_$2_$wl.json 2> /dev/null
    python -c "
import json; d=json.loads(open('gpurun_out/o_$1_$2_$wl.json').read().strip().splitlines()[-1]); print('occ $1 $2 $wl', '%.3f'%d['ms_per_step'], {k:round(v['ms'],3) for k,v in d['roofline']['kernels'].items()})"
  done
done
