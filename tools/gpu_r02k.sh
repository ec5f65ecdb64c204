# round-2 HEAD measurement: GPU suite, smoke, C3 launch list (ncu phases -> roofline traffic), the
# default bench line (driver command), the reference arm, and every config's bench line
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
lscpu > gpurun_out/lscpu.txt 2>&1; nproc > gpurun_out/nproc.txt
if [ -z "$NOTEST" ]; then
  timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/gpu_tests.log
  timeout 300 python __graft_entry__.py smoke > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
fi
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 1200 --csv \
  --log-file gpurun_out/launches_C3.csv python bench.py --config C3 --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch.log 2>&1
python tools/ncu_phases.py gpurun_out/launches_C3.csv C3 6 gpurun_out/ncu_phases_C3.json > /dev/null 2>&1 && cp gpurun_out/ncu_phases_C3.json profiles/
timeout 900 python bench.py > gpurun_out/bench_default.log 2>&1
timeout 900 python bench.py --impl reference > gpurun_out/bench_reference.log 2>&1
for c in C1 C2 C4a C4b C5; do
  timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.log 2>&1
done
timeout 300 python bench.py --config C5 --rle on --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_C5rle.log 2>&1
timeout 300 python bench.py --config C2 --rle auto --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_C2auto.log 2>&1
true
