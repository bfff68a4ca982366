# One GPU session: build, GPU tests, smoke, default bench, then optional sweep points ($@).
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
eval timeout 1500 python -m pytest tests -m gpu -x -q ${NM_TESTS:-} > gpurun_out/gpu_tests.log 2>&1; echo tests_rc=$?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke_rc=$?
timeout 600 python bench.py > gpurun_out/bench.log 2>&1; echo bench_rc=$?
if [ -n "$NM_SWEEP" ]; then timeout 2400 python tools/sweep.py gpurun_out/sweep_c2.jsonl $NM_SWEEP > gpurun_out/sweep.log 2>&1; echo sweep_rc=$?; fi
