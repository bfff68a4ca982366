set -x
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
(cd tools/probes && nvcc -gencode arch=compute_100a,code=sm_100a -O2 -o probe_sparse_peak probe_sparse_peak.cu && timeout 120 ./probe_sparse_peak) > gpurun_out/probe_sparse_peak.txt 2>&1; tail -4 gpurun_out/probe_sparse_peak.txt
timeout 900 python -m pytest tests/test_parity_pack_spmm.py -x -q -k "residual or spmm or formats" > gpurun_out/t_dbg.log 2>&1; echo tests=$?; tail -15 gpurun_out/t_dbg.log
timeout 600 compute-sanitizer --tool memcheck --print-limit 10 python tools/sanitize_spmm.py > gpurun_out/san_dbg.log 2>&1; echo san=$?; head -40 gpurun_out/san_dbg.log
timeout 900 python -m pytest tests/test_parity_models.py -x -q > gpurun_out/t_models.log 2>&1; echo models=$?; tail -15 gpurun_out/t_models.log
