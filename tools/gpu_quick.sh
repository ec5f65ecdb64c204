# quick GPU check: gpu tests (unless NOTEST=1) + short benches of $CFGS (default C3)
CFGS=${CFGS:-C3}
if [ -z "$NOTEST" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
fi
for c in $CFGS; do
  timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
done
