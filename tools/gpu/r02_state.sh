# round-2 re-entry: health check + headline measurement of the committed state
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/gpu.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?; tail -3 gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/r02_bench_c3.json 2> gpurun_out/r02_bench_c3.err; echo bench=$?; tail -c 3000 gpurun_out/r02_bench_c3.json
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider --durations=25 > gpurun_out/gpu_tests.log 2>&1; echo tests=$?; tail -40 gpurun_out/gpu_tests.log
for wl in c3-reddit-f128-128:2:16 c4-proteins-f256-128:2:16 c5-products-f100-128:2:8 c2-banded-n1m-d16-f128-1:2:4; do
  timeout 900 python bench.py --workload $wl --no-cpu --steps 30 > gpurun_out/r02_bench_$wl.json 2> gpurun_out/r02_bench_$wl.err; echo $wl=$?
done
