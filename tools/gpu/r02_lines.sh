set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
for wl in c4-proteins-f256-128:2:16 c5-products-f100-128:2:8 c3-reddit-f128-128:2:16; do
  timeout 900 python bench.py --workload $wl --steps 30 > gpurun_out/z_bench_$wl.json 2> gpurun_out/z_bench_$wl.err; echo $wl=$?
done
