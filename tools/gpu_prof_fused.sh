# fused-pass profiling: quick tests, a C3 bench, ncu launch list + one --set full capture of k_fused
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 200 python -m pytest tests/test_gpu_parity.py -q -x -k fused > gpurun_out/fused_tests.log 2>&1; echo "rc=$?" >> gpurun_out/fused_tests.log
for c in ${CFGS:-C3}; do timeout 150 python bench.py --config $c --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1; done
timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 200 --csv \
  --log-file gpurun_out/launches_C3.csv python bench.py --config C3 --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch.log 2>&1
timeout 400 ncu --set full --import-source on --clock-control none -k regex:k_fused -s 1 -c 1 -o gpurun_out/full_fused -f \
  python bench.py --config C3 --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full.log 2>&1
