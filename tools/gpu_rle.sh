# RLE run split: RLE-related GPU tests + C5/C2 benches (RLE on, run split on/off, plain) + launch lists
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 900 python -m pytest tests -m gpu -x -q -k "rle or RLE or invariants" > gpurun_out/rle_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/rle_tests.log
timeout 300 python bench.py --config C5 --rle on --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_C5rle.log 2>&1
GBDT_RUNSPLIT=0 timeout 300 python bench.py --config C5 --rle on --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_C5rle_scan.log 2>&1
timeout 300 python bench.py --config C2 --rle auto --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/bench_C2auto.log 2>&1
for c in C5 C2; do
timeout 400 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -c 1500 --csv \
  --log-file gpurun_out/launches_${c}rle.csv python bench.py --config $c --rle ${RLEMODE:-auto} --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch_rle.log 2>&1
done
true
