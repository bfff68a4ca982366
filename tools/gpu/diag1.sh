set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
B="timeout 600 python bench.py --no-cpu --no-cusparse --steps 30"
for wl in c2-banded-n1m-d16-f128-1:2:4 c2-banded-n1m-d16-f128-1:2:4-tau0; do
  $B --workload $wl 2>&1 | tail -1 > gpurun_out/d_$wl.json
  NM_SPMM_DEBUG=32 $B --workload $wl 2>&1 | tail -1 > gpurun_out/d32_$wl.json
  NM_SPMM_DEBUG=1 $B --workload $wl 2>&1 | tail -1 > gpurun_out/d1_$wl.json
  NM_SPMM_DEBUG=2 $B --workload $wl 2>&1 | tail -1 > gpurun_out/d2_$wl.json
  timeout 300 python tools/trace_spmm.py $wl > gpurun_out/trace_$wl.txt 2>&1
done
