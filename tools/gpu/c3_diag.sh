# sparse-MMA peak probe + k_spmm_sptc attribution (NM_SPMM_DEBUG) + ncu of both kernels on C3
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
(cd tools/probes && nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o probe_sparse_peak probe_sparse_peak.cu && timeout 300 ./probe_sparse_peak) > gpurun_out/probe_sparse_peak.txt 2>&1
tail -3 gpurun_out/probe_sparse_peak.txt
WL=c3-reddit-f128-1:2:4
ID="--max-outer 0 --max-stage1 -1 --max-stage2 -1"
for dbg in 0 2 128 64 192 1120; do
  NM_SPMM_DEBUG=$dbg timeout 600 python bench.py --no-cpu --no-cusparse --steps 10 --workload $WL $ID > gpurun_out/c3dbg_$dbg.json 2> gpurun_out/c3dbg_$dbg.err
  python - gpurun_out/c3dbg_$dbg.json <<'PY'
import json,sys
d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); k=d['roofline']['kernels']
print(sys.argv[1], ' '.join('%s %.3f'%(n,v['ms']) for n,v in k.items()), 'chunks', d['preprocess']['n_chunks'])
PY
done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_sptc -s 3 -c 1 -o gpurun_out/c3_sptc python bench.py --no-cpu --no-cusparse --steps 1 --warmup 3 --workload $WL $ID > gpurun_out/ncu1.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_residual -s 3 -c 1 -o gpurun_out/c3_res python bench.py --no-cpu --no-cusparse --steps 1 --warmup 3 --workload $WL $ID > gpurun_out/ncu2.log 2>&1
ls -la gpurun_out
