# MMA issue-loop feature probe, bulk-vs-cp.async gather probe, V_p = 64 parity tests
set -x
timeout 300 tools/probes/probe_mma_issue > gpurun_out/probe_mma_issue2.txt 2>&1; echo probe=$?; cat gpurun_out/probe_mma_issue2.txt
timeout 300 tools/probes/probe_bulk_gather > gpurun_out/probe_bulk_gather.txt 2>&1; echo probe2=$?; cat gpurun_out/probe_bulk_gather.txt
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 1500 python -m pytest tests/test_parity_pack_spmm.py tests/test_parity_gnn_fullsize.py tests/test_abi.py -q -x --timeout 900 -p no:cacheprovider -k "not bench_launch" > gpurun_out/t_vp.log 2>&1; echo tests=$?; tail -15 gpurun_out/t_vp.log
