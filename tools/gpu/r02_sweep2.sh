set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python bench.py > gpurun_out/s_bench_c3.json 2> gpurun_out/s_bench_c3.err; echo bench=$?; tail -c 300 gpurun_out/s_bench_c3.json
for wl in c4-proteins-f256-128:2:16 c5-products-f100-128:2:8 c3-reddit-f128-128:2:16; do
  timeout 1200 python bench.py --workload $wl --steps 30 > gpurun_out/s_bench_$wl.json 2> gpurun_out/s_bench_$wl.err; echo $wl=$?
done
timeout 3600 python tools/sweep.py gpurun_out/s_sweep_c2.jsonl > gpurun_out/s_sweep_c2.txt 2>&1; echo sweep=$?; tail -20 gpurun_out/s_sweep_c2.txt
