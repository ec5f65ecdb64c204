# GPU: C4b graph vs eager, short path on/off, 20 trees; short-path tests
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 600 python -m pytest tests/test_gpu_short.py -q -x > gpurun_out/short_tests.log 2>&1; echo "rc=$?" >> gpurun_out/short_tests.log
for c in ${CFGS:-C4b}; do
for gr in 1 0; do for s in 1 0; do
  GBDT_GRAPH=$gr GBDT_SHORT=$s timeout 200 python bench.py --config $c --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_g${gr}_s${s}_$c.log 2>&1
done; done; done
