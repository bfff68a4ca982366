set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_parity_gcn.py tests/test_dist_gpu.py -q -p no:cacheprovider > gpurun_out/t_fused.log 2>&1; echo tfused=$?; tail -5 gpurun_out/t_fused.log
bash tools/gpu/r02_groups.sh
