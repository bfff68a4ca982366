# round-2 measurement run: every GPU test, smoke, headline + per-config bench lines, launch list,
# configs[1] sweep, GCN layer timing, reorder timing
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv > gpurun_out/m_gpu.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 2400 python -m pytest tests -m gpu -q --timeout 1200 -p no:cacheprovider --durations=15 > gpurun_out/m_gpu_tests.log 2>&1; echo tests=$?; tail -22 gpurun_out/m_gpu_tests.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/m_smoke.log 2>&1; echo smoke=$?; tail -3 gpurun_out/m_smoke.log
timeout 1200 python bench.py > gpurun_out/m_bench_c3.json 2> gpurun_out/m_bench_c3.err; echo bench=$?; tail -c 400 gpurun_out/m_bench_c3.json
timeout 600 python bench.py --impl reference --steps 5 --warmup 3 > gpurun_out/m_bench_ref.json 2> gpurun_out/m_bench_ref.err; echo ref=$?; tail -c 300 gpurun_out/m_bench_ref.json
for wl in c3-reddit-f128-128:2:16 c4-proteins-f256-128:2:16 c5-products-f100-128:2:8 c1-er-n2048-f32-1:2:4; do
  timeout 1200 python bench.py --workload $wl --steps 30 > gpurun_out/m_bench_$wl.json 2> gpurun_out/m_bench_$wl.err; echo $wl=$?
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 3000 --csv --log-file gpurun_out/m_launches_c3.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-cusparse > gpurun_out/m_launches_bench.log 2>&1; echo launches=$?
timeout 1800 python tools/gcn_timing.py gpurun_out/m_gcn_layers.jsonl > gpurun_out/m_gcn_timing.log 2>&1; echo gcn=$?; tail -5 gpurun_out/m_gcn_timing.log
timeout 3600 python tools/sweep.py gpurun_out/m_sweep_c2.jsonl > gpurun_out/m_sweep_c2.txt 2>&1; echo sweep=$?; tail -20 gpurun_out/m_sweep_c2.txt
timeout 1800 python tools/reorder_timing.py gpurun_out/m_reorder_timing.jsonl > gpurun_out/m_reorder_timing.log 2>&1; echo reorder=$?; tail -12 gpurun_out/m_reorder_timing.log
