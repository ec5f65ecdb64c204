# GPU: all gpu tests + smoke, then SmartGD on/off (Fig. 9 ablation) on C2 and C3 (20 trees each)
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
for c in C2 C3; do
  for s in on off; do
    timeout 600 python bench.py --config $c --steps 20 --warmup 3 --smartgd $s --no-e2e --no-cpu-baseline > gpurun_out/bench_sgd${s}_$c.log 2>&1
  done
done
