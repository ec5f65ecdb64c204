# GPU: gpu tests (TESTS=1); graph vs eager on the latency-bound configs; depth
# sweep 2-8 on C2 and C3; tree-count sweep 10-80 on C2
if [ -n "$TESTS" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
fi
B="timeout 600 python bench.py --warmup 3 --no-e2e --no-cpu-baseline"
for c in C1 C4b C2 C3; do
  $B --config $c --steps 20 > gpurun_out/bench_graph_$c.log 2>&1
  GBDT_GRAPH=0 $B --config $c --steps 20 > gpurun_out/bench_eager_$c.log 2>&1
done
for d in 2 3 4 5 6 7 8; do
  $B --config C2 --steps 20 --depth $d > gpurun_out/sweep_depth${d}_C2.log 2>&1
  $B --config C3 --steps 10 --depth $d > gpurun_out/sweep_depth${d}_C3.log 2>&1
done
for T in 10 20 40 80; do
  $B --config C2 --steps $T > gpurun_out/sweep_trees${T}_C2.log 2>&1
done
