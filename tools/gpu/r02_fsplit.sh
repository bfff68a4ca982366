# F-slab split experiment on C3/C4 (L2 working set) + ncu of k_residual on C5
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1200 python tools/fsplit_exp.py c3-reddit-f128-1:2:4 c4-proteins-f256-128:2:16 c5-products-f100-128:2:8 > gpurun_out/fsplit.jsonl 2> gpurun_out/fsplit.err; echo fsplit=$?; cat gpurun_out/fsplit.jsonl; tail -3 gpurun_out/fsplit.err
timeout 1200 ncu --set full --clock-control none -k regex:"k_residual|k_spmm_full" -s 4 -c 2 -o gpurun_out/r02_c5 -f \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-cusparse --layout natural --no-reorder --workload c5-products-f100-128:2:8 > gpurun_out/r02_ncu_c5.log 2>&1; echo ncu=$?
