set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python bench.py > gpurun_out/h_bench_c3.json 2> gpurun_out/h_bench_c3.err; echo bench=$?; tail -c 400 gpurun_out/h_bench_c3.json
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/h_bench_ref.json 2> gpurun_out/h_bench_ref.err; echo ref=$?
for wl in c4-proteins-f256-128:2:16 c2-banded-n1m-d16-f128-1:2:4; do
  timeout 1200 python bench.py --workload $wl --steps 30 > gpurun_out/h_bench_$wl.json 2> gpurun_out/h_bench_$wl.err; echo $wl=$?
done
