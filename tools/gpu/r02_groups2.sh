set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_parity_gcn.py tests/test_dist_gpu.py -q -p no:cacheprovider > gpurun_out/t_fused.log 2>&1; echo tfused=$?; tail -5 gpurun_out/t_fused.log
bash tools/gpu/r02_groups.sh
python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > gpurun_out/build_default.log 2>&1
for tool in memcheck synccheck racecheck; do
  timeout 1200 compute-sanitizer --tool $tool --print-limit 20 python tools/sanitize_spmm.py > gpurun_out/r02_sanitize_$tool.log 2>&1; echo $tool rc=$?; tail -4 gpurun_out/r02_sanitize_$tool.log
done
