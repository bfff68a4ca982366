# Tuning experiments on the GPU box: build the package with extra -D flags into _alt/<name>
# and run bench.py there.  Usage: variants.sh "<wl1> <wl2>" name1:"-DA=1" name2:"-DB=2" ...
WLS="$1"; shift
for spec in "$@"; do
  name="${spec%%:*}"; flags="${spec#*:}"
  d=_alt/$name; rm -rf $d; mkdir -p $d
  cp -r paper_conf_ppopp_chensz0s25_b200 oracle include bench_support bench.py __graft_entry__.py $d/
  rm -f $d/paper_conf_ppopp_chensz0s25_b200/libnm.so
  (cd $d && NM_NVCC_FLAGS="$flags" python -c "from paper_conf_ppopp_chensz0s25_b200 import build; build.build(force=True)" > build.log 2>&1) || { echo "$name build failed"; cat $d/build.log | tail -5; continue; }
  for wl in $WLS; do
    (cd $d && timeout 600 python bench.py --no-cpu --no-cusparse --steps 30 --workload $wl 2>&1 | tail -1 | python -c "
import json,sys
d=json.loads(sys.stdin.read()); k=d['roofline']['kernels']
print('%-8s %-40s %8.0f GF/s  step %.3f ms  ' % ('$name', '$wl', d['value'], d['ms_per_step']) + '  '.join('%s %.3fms/%.2f' % (n, v['ms'], v['frac']) for n, v in k.items()))
" ) || echo "$name $wl FAILED"
  done
done
