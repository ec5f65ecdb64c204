make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_invariants.py -q -x > gpurun_out/dsm_tests.log 2>&1; echo "rc=$?" >> gpurun_out/dsm_tests.log
for c in C3 C5 C2; do
  timeout 150 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_dsm_$c.log 2>&1
  GBDT_DSM=0 timeout 150 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_l1_$c.log 2>&1
done
