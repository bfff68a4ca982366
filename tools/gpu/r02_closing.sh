# closing check on the final code: every GPU test, smoke, headline bench
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider --durations=10 > gpurun_out/c_gpu_tests.log 2>&1; echo tests=$?; tail -15 gpurun_out/c_gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/c_smoke.log 2>&1; echo smoke=$?; tail -3 gpurun_out/c_smoke.log
timeout 1200 python bench.py > gpurun_out/c_bench_c3.json 2> gpurun_out/c_bench_c3.err; echo bench=$?; tail -c 400 gpurun_out/c_bench_c3.json
