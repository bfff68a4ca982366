# ncu evidence for one bench workload: launch list + one full capture of the SpMM kernel.
# usage: prof.sh <workload> <tag>
WL=${1:-c2-banded-n1m-d16-f128-1:2:4}; TAG=${2:-cur}
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_$TAG.csv \
  python bench.py --steps 5 --warmup 3 --no-cpu --no-cusparse --workload $WL > gpurun_out/launch_bench_$TAG.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_spmm_sptc -s 3 -c 1 -o gpurun_out/prof_$TAG -f \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-cusparse --workload $WL > gpurun_out/prof_bench_$TAG.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_residual -s 3 -c 1 -o gpurun_out/profres_$TAG -f \
  python bench.py --steps 2 --warmup 3 --no-cpu --no-cusparse --workload $WL > gpurun_out/profres_bench_$TAG.log 2>&1
echo done
