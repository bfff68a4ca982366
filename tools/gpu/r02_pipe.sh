# residual batches pipelined across items (k_residual_p) vs k_residual: parity + A/B
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/test_parity_pack_spmm.py tests/test_parity_fullsize.py tests/test_parity_models.py tests/test_parity_gcn.py -q -x --timeout 900 -p no:cacheprovider > gpurun_out/t_pipe.log 2>&1; echo tests=$?; tail -4 gpurun_out/t_pipe.log
for pipe in 1 0; do
  NM_NVCC_FLAGS="-DNM_RES_PIPE=$pipe" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/build_p$pipe.log 2>&1
  for wl in c3-reddit-f128-1:2:4 c4-proteins-f256-128:2:16 c5-products-f100-128:2:8 c2-banded-n262k-d16-f128-64:2:8 c2-powerlaw-n262k-d16-f128-1:2:4 c2-powerlaw-n65k-d8-f128-1:2:4; do
    timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl --layout natural --no-reorder --sptc-format 1 > gpurun_out/p${pipe}_$wl.json 2> /dev/null
    python -c "
import json; d=json.loads(open('gpurun_out/p${pipe}_$wl.json').read().strip().splitlines()[-1]); print('pipe $pipe $wl', '%.3f'%d['ms_per_step'], {k:round(v['ms'],3) for k,v in d['roofline']['kernels'].items()})"
  done
done
