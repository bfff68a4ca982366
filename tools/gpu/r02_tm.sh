# compressed records with A in tensor memory (format 3): parity, then A/B vs full records
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python -m pytest tests/test_parity_pack_spmm.py tests/test_parity_gcn.py tests/test_parity_models.py tests/test_score_patterns.py tests/test_dist_gpu.py -q --timeout 600 -p no:cacheprovider -k "formats_agree or panel_height or conforming or gcn or sgc or sage or cheb or score or bcast or fused" > gpurun_out/t_tm.log 2>&1; echo tests=$?; tail -15 gpurun_out/t_tm.log
summ() { python - $1 <<'PY'
import json,sys
try:
    d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']; pp=d['preprocess']
    print(sys.argv[1].split('/')[-1], 'step %.3f'%d['ms_per_step'], '%.0f GF/s'%d['value'], ' '.join('%s %.3f (%s %.2f)'%(n,v['ms'],v['bound'],v['frac']) for n,v in k.items()))
except Exception as e: print(sys.argv[1], 'FAIL', e)
PY
}
for wl in c2-banded-n1m-d16-f128-1:2:4 c3-reddit-f128-1:2:4 c4-proteins-f256-128:2:16 c2-banded-n262k-d16-f128-64:2:8 c2-powerlaw-n262k-d16-f128-1:2:4; do
  for fmt in 1 3; do
    timeout 900 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl --sptc-format $fmt --layout natural --no-reorder > gpurun_out/tm${fmt}_$wl.json 2> gpurun_out/tm${fmt}_$wl.err
    summ gpurun_out/tm${fmt}_$wl.json
  done
done
for xp in 8 16 32; do
  timeout 900 python bench.py --no-cpu --no-cusparse --steps 20 --workload c5-products-f100-128:2:8 --layout natural --no-reorder --xpad $xp > gpurun_out/xpad${xp}_c5.json 2> gpurun_out/xpad${xp}_c5.err
  summ gpurun_out/xpad${xp}_c5.json
done
