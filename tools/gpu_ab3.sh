make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 1500 python -m pytest tests -m gpu -x -q -k "not fullsize" > gpurun_out/ab3_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/ab3_tests.log
for c in C3 C4a C2; do timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ab3_$c.log 2>&1; done
true
