# round-2 measurements: regression tests, headline + per-config bench lines, launch list, ncu, sweep, GCN layers
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1800 python -m pytest tests/test_parity_pack_spmm.py tests/test_parity_models.py tests/test_parity_gnn_fullsize.py -q --timeout 900 -p no:cacheprovider > gpurun_out/t_final.log 2>&1; echo tests=$?; tail -4 gpurun_out/t_final.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout 1200 python bench.py > gpurun_out/r02_bench_c3.json 2> gpurun_out/r02_bench_c3.err; echo bench=$?; tail -c 600 gpurun_out/r02_bench_c3.json
for wl in c3-reddit-f128-128:2:16 c4-proteins-f256-128:2:16 c5-products-f100-128:2:8 c2-banded-n1m-d16-f128-1:2:4; do
  timeout 1200 python bench.py --workload $wl --no-cpu --steps 50 > gpurun_out/r02_bench_$wl.json 2> gpurun_out/r02_bench_$wl.err; echo $wl=$?
done
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none -c 4000 --csv --log-file gpurun_out/r02_launches_c3.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-cusparse > gpurun_out/r02_launches_bench.log 2>&1; echo launches=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_spmm_full|k_residual" -s 6 -c 2 -o gpurun_out/r02_c3_final python bench.py --no-cpu --no-cusparse --steps 1 --warmup 3 --no-reorder --layout reordered > gpurun_out/ncu_final.log 2>&1; echo ncu=$?
timeout 3000 python tools/sweep.py gpurun_out/sweep_c2.jsonl > gpurun_out/sweep_c2.txt 2>&1; echo sweep=$?; tail -20 gpurun_out/sweep_c2.txt
timeout 1800 python tools/gcn_timing.py gpurun_out/r02_gcn_layers.jsonl > gpurun_out/gcn_timing.log 2>&1; echo gcn=$?; tail -5 gpurun_out/gcn_timing.log
