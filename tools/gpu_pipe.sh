# pipelined local shards: GPU tests that use several local shards, then C3/C2/C5 benches A/B
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 1200 python -m pytest tests -m gpu -x -q -k "shard or Shard" > gpurun_out/pipe_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/pipe_tests.log
for c in ${CFGS:-C3 C2 C5}; do for k in 2 4; do
  timeout 300 python bench.py --config $c --local-shards $k --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_${c}_p$k.log 2>&1
  GBDT_PIPE=0 timeout 300 python bench.py --config $c --local-shards $k --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_${c}_s$k.log 2>&1
done; done
true
