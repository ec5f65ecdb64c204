make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 600 python -m pytest tests/test_gpu_invariants.py tests/test_gpu_next.py -q -x > gpurun_out/inv_tests.log 2>&1; echo "rc=$?" >> gpurun_out/inv_tests.log
