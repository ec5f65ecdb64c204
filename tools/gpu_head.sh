# HEAD check on a fresh box: gpu tests, smoke, short benches of every config (RLE on/off for C5)
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
if [ -z "$NOTEST" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
  timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
fi
for c in ${CFGS:-C3 C2 C4a C4b C5}; do
  timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
done
[ -n "$RLE5" ] && timeout 300 python bench.py --config C5 --rle on --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_C5rle.log 2>&1
true
