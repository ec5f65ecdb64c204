# single-pass scans: full GPU suite, then every config's bench with the look-back scan and the
# three-phase scan (GBDT_SCAN3=1)
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 1800 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
for c in C2 C3 C4a C4b C5; do
  timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
  GBDT_SCAN3=1 timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_${c}_s3.log 2>&1
done
timeout 300 python bench.py --config C5 --rle on --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_C5rle.log 2>&1
GBDT_SCAN3=1 timeout 300 python bench.py --config C5 --rle on --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_C5rle_s3.log 2>&1
true
