set -x
(cd tools/probes && nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o probe_sparse_peak probe_sparse_peak.cu && timeout 120 ./probe_sparse_peak) > gpurun_out/probe_sparse_peak.txt 2>&1
tail -5 gpurun_out/probe_sparse_peak.txt
for v in 1 0; do
  NM_NVCC_FLAGS="-DNM_RES_CPASYNC=$v" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/bld_res$v.log 2>&1
  timeout 900 python -m pytest tests/test_parity_pack_spmm.py -x -q -k "formats or concurrent or residual_split" > gpurun_out/t_res$v.log 2>&1; echo tests$v=$?; tail -2 gpurun_out/t_res$v.log
  for wl in c3-reddit-f128-1:2:4 c5-products-f100-128:2:8 c2-banded-n1m-d16-f128-1:2:4; do
    timeout 900 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl --max-outer 0 --max-stage1 -1 --max-stage2 -1 > gpurun_out/rc${v}_$wl.json 2> gpurun_out/rc${v}_$wl.err
    python - gpurun_out/rc${v}_$wl.json <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']; pp=d['preprocess']
    print(sys.argv[1], '%.0f GF/s'%d['value'], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()), 'res', pp['residual_nnz'])
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
  done
done
