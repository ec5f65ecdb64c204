# full GPU suite + smoke + C3/C2/C5/C4a benches
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
for c in ${CFGS:-C3 C2 C5 C4a}; do timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/full_$c.log 2>&1; done
true
