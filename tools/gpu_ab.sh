# GPU: tests (unless NOTEST=1), then C3/C2/C5 benches with the fused and the 3-pass partition
if [ -z "$NOTEST" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
fi
for c in ${CFGS:-C3 C2 C5}; do
  timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
  GBDT_PARTITION=3pass timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench3p_$c.log 2>&1
done
