make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 1500 python -m pytest tests/test_gpu_fullsize_parity.py -m gpu -q -x -s --durations=10 > gpurun_out/fullsize_parity.log 2>&1; echo "tests rc=$?" >> gpurun_out/fullsize_parity.log
