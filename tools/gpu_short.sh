# GPU: short-list path -- its tests + sparse parity tests, C4a/C4b benches with GBDT_SHORT=0 / 1,
# optional full-size parity ($FULL = -k expression) and C4a launch list ($LAUNCH)
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 900 python -m pytest tests/test_gpu_short.py tests/test_gpu_parity.py tests/test_gpu_invariants.py tests/test_gpu_variants.py tests/test_gpu_next.py -q -x ${TK:+-k "$TK"} > gpurun_out/short_tests.log 2>&1; echo "rc=$?" >> gpurun_out/short_tests.log
for c in ${CFGS:-C4a C4b}; do
  for s in ${SHORTS:-0 1}; do
    GBDT_SHORT=$s $BENV timeout 200 python bench.py --config $c --steps ${STEPS:-5} --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_short${s}_$c.log 2>&1
  done
done
if [ -n "$LAUNCH" ]; then
  timeout 400 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -c 1200 --csv \
    --log-file gpurun_out/launches_C4a.csv python bench.py --config C4a --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch.log 2>&1
fi
if [ -n "$FULL" ]; then
  timeout 900 python -m pytest tests/test_gpu_fullsize_parity.py -q -x -k "$FULL" > gpurun_out/short_full.log 2>&1; echo "rc=$?" >> gpurun_out/short_full.log
fi
