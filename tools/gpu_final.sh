# GPU: gpu tests + smoke, the default bench line (C3 with e2e + cpu_baseline), per-config lines,
# and the C3 launch list + full ncu captures of the streaming kernels (tools/profile_round.sh)
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 900 python bench.py > gpurun_out/bench_default.log 2>&1
for c in C1 C2 C4a C4b C5; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
done
timeout 600 python bench.py --config C5 --rle on --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_C5rle.log 2>&1
if [ -z "$NOPROF" ]; then CFG=C3 bash tools/profile_round.sh; fi
