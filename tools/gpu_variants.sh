# GPU: C3 (or $CFGS) bench for the default library and each variant libgbdt_<V>.so ($VARIANTS)
for c in ${CFGS:-C3}; do
  timeout 300 python bench.py --config $c --steps ${STEPS:-10} --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_base_$c.log 2>&1
  for v in $VARIANTS; do
    GBDT_LIB=$PWD/paper_conf_ipps_wenhkls18_b200/libgbdt_$v.so timeout 300 python bench.py --config $c --steps ${STEPS:-10} --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_${v}_$c.log 2>&1
  done
done
