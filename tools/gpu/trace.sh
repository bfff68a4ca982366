# clock64 timeline of CTA 0 for one workload: builds a trace-enabled copy under _alt/trace
WL=${1:-c2-banded-n1m-d16-f128-1:2:4}
d=_alt/trace; rm -rf $d; mkdir -p $d
cp -r paper_conf_ppopp_chensz0s25_b200 oracle include bench_support bench.py tools $d/
rm -f $d/paper_conf_ppopp_chensz0s25_b200/libnm.so
(cd $d && NM_NVCC_FLAGS="-DNM_SPMM_TRACE_BUILD" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > build.log 2>&1) || { echo "trace build failed"; tail -5 $d/build.log; exit 1; }
(cd $d && timeout 300 python tools/trace_spmm.py $WL)
