# final round-2 evidence with nm_pack_auto: headline bench, launch list (SpMM kernels), configs[1] sweep
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python bench.py > gpurun_out/f_bench_c3.json 2> gpurun_out/f_bench_c3.err; echo bench=$?; tail -c 300 gpurun_out/f_bench_c3.json
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_spmm|k_residual" -c 40 --csv --log-file gpurun_out/f_launches_c3.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-cusparse --no-reorder --layout natural > gpurun_out/f_launches_bench.log 2>&1; echo launches=$?
timeout 3600 python tools/sweep.py gpurun_out/f_sweep_c2.jsonl > gpurun_out/f_sweep_c2.txt 2>&1; echo sweep=$?; tail -20 gpurun_out/f_sweep_c2.txt
