# missing-value split path: GPU tests touching missing values / sparse data + C4a/C4b benches A/B
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 1200 python -m pytest tests -m gpu -x -q -k "missing or sparse or c4 or C4 or short or nan or random or edge or rle" > gpurun_out/miss_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/miss_tests.log
for c in C4a C4b; do
timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
GBDT_FASTMISS=0 timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_${c}_gen.log 2>&1
done
true
