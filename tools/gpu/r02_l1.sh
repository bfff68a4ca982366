# residual X gathers through L1 (cp.async.ca) vs bypass, C3/C4/C5 (residual kernel only, fsplit tool's full_* numbers)
set -x
for v in 0 1 2; do
  NM_NVCC_FLAGS="-DNM_RES_L1=$v" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/build_l1$v.log 2>&1
  FSPLIT=0 timeout 900 python tools/fsplit_exp.py c3-reddit-f128-1:2:4 c4-proteins-f256-128:2:16 c5-products-f100-128:2:8 > gpurun_out/l1_$v.jsonl 2> gpurun_out/l1_$v.err; echo v$v=$?
  python -c "
import json
for l in open('gpurun_out/l1_$v.jsonl'):
    d=json.loads(l); print('L1=$v', d['workload'], 'full %.3f sptc %.3f res %.3f' % (d['full_ms'], d['full_sptc_ms'], d['full_res_ms']))"
done
