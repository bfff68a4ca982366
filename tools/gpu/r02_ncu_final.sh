# ncu evidence on the final code: launch list of the bench command (SpMM kernels) + full captures of both kernels on C3
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_spmm|k_residual" -c 40 --csv --log-file gpurun_out/fin_launches_c3.csv python bench.py --steps 5 --warmup 3 --no-cpu --no-cusparse --no-reorder --layout natural > gpurun_out/fin_launches.log 2>&1; echo launches=$?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_spmm_full|k_residual" -s 4 -c 2 -o gpurun_out/fin_c3 -f \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-cusparse --layout natural --no-reorder --sptc-format 1 > gpurun_out/fin_ncu.log 2>&1; echo ncu=$?
