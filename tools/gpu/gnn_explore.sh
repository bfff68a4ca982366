# C3-C5 (GNN-shaped) bench lines with capped reorders: preprocessing times, residual share,
# kernel times and cuSPARSE on one box.  usage: bash tools/gpu/gnn_explore.sh
set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
run() { tag=$1; shift; NM_REORDER_TRACE=1 timeout ${TMO:-900} python bench.py --no-cpu --steps 20 "$@" > gpurun_out/gx_$tag.json 2> gpurun_out/gx_$tag.err; echo "$tag rc=$?"; tail -c 600 gpurun_out/gx_$tag.json; }
run c3_124_o1s0 --workload c3-reddit-f128-1:2:4 --max-outer 1 --max-stage2 0
run c3_124_o1s0_tau8 --workload c3-reddit-f128-1:2:4 --max-outer 1 --max-stage2 0 --tau 8 --no-cusparse
run c3_12816_o1s0 --workload c3-reddit-f128-128:2:16 --max-outer 1 --max-stage2 0 --no-cusparse
run c4_o1s0 --workload c4-proteins-f256-128:2:16 --max-outer 1 --max-stage2 0
run c5_o1s0 --workload c5-products-f100-128:2:8 --max-outer 1 --max-stage2 0
run c3_124_o1s1 --workload c3-reddit-f128-1:2:4 --max-outer 1 --max-stage2 1 --no-cusparse
