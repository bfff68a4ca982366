set -x
for kb in 96 16 4; do
  NM_NVCC_FLAGS="-DNM_TM_PF_KB=$kb" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/build_tmpf.log 2>&1
  for wl in c3-reddit-f128-1:2:4 c2-banded-n1m-d16-f128-1:2:4 c5-products-f100-128:2:8; do
    timeout 600 python bench.py --no-cpu --no-cusparse --steps 30 --workload $wl --layout natural --no-reorder --sptc-format 3 > gpurun_out/tmpf_${kb}_$wl.json 2> /dev/null
    python -c "
import json; d=json.loads(open('gpurun_out/tmpf_${kb}_$wl.json').read().strip().splitlines()[-1]); print('tmpf $kb $wl', '%.3f'%d['ms_per_step'], {k:round(v['ms'],3) for k,v in d['roofline']['kernels'].items()})"
  done
done
