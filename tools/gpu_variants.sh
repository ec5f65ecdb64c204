# GPU: gpu tests (TESTS=1), then C3 (or $CFGS) bench for the default library and each variant
# libgbdt_<V>.so ($VARIANTS); extra bench args in $BARGS
if [ -n "$TESTS" ]; then
  timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
fi
for c in ${CFGS:-C3}; do
  timeout 150 python bench.py --config $c --steps ${STEPS:-10} --warmup 3 --no-e2e --no-cpu-baseline $BARGS > gpurun_out/bench_base_$c.log 2>&1
  for v in $VARIANTS; do
    GBDT_LIB=$PWD/paper_conf_ipps_wenhkls18_b200/libgbdt_$v.so timeout 150 python bench.py --config $c --steps ${STEPS:-10} --warmup 3 --no-e2e --no-cpu-baseline $BARGS > gpurun_out/bench_${v}_$c.log 2>&1
  done
done
