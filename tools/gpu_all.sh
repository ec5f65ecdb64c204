# GPU: tests + one bench line per config (RLE on for C5 as a second line)
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
for c in C3 C2 C5 C4a C4b C1; do
  timeout 300 python bench.py --config $c --steps ${STEPS:-10} --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
done
timeout 300 python bench.py --config C5 --rle on --steps ${STEPS:-10} --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_C5rle.log 2>&1
