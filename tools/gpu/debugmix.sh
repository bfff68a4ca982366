# time k_spmm_sptc under NM_SPMM_DEBUG switches (results invalid; critical-path attribution)
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for wl in ${WLS:-c2-banded-n1m-d16-f128-1:2:4-tau0}; do
for dbg in ${DBGS:-0 2 16 32 64 128 192 256 66 194 450}; do
  NM_SPMM_DEBUG=$dbg timeout 600 python bench.py --no-cpu --no-cusparse --steps 20 --workload $wl 2>&1 | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read()); k=d['roofline']['kernels']
print('dbg=%-4s %-40s sptc %.3f ms' % ('$dbg', '$wl', k['k_spmm_sptc']['ms']))" || echo "dbg=$dbg failed"
done
done
