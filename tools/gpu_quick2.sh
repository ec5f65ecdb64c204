# quick check: fused parity tests + short benches of $CFGS (env $BENV applied to the benches)
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 200 python -m pytest tests/test_gpu_parity.py -q -x -k fused > gpurun_out/fused_tests.log 2>&1; echo "rc=$?" >> gpurun_out/fused_tests.log
for c in ${CFGS:-C3 C2 C5}; do env $BENV timeout 150 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
