make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
nproc > gpurun_out/host.txt; lscpu >> gpurun_out/host.txt
timeout 1100 python -m pytest tests -m gpu -q -x --durations=15 > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
timeout 300 python bench.py --config C3 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_C3.log 2>&1
