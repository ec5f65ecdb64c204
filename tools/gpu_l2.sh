# GPU: gpu tests, then C3/C2/C5 with and without the L2 persisting window (GBDT_L2_PERSIST=0)
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
for c in C3 C2 C5; do
  timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_l2on_$c.log 2>&1
  GBDT_L2_PERSIST=0 timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_l2off_$c.log 2>&1
done
K=k_chunk_agg S=0 TAG=l2 bash tools/ncu_one.sh
