# GPU: default bench line (C3 with e2e + cpu_baseline), the C3 launch list + full ncu captures of the
# streaming kernels (tools/profile_round.sh), and a C4a launch list
timeout 900 python bench.py > gpurun_out/bench_default.log 2>&1
CFG=C3 bash tools/profile_round.sh
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    -c 2000 --csv --log-file gpurun_out/launches_C4a.csv \
    python bench.py --config C4a --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch_C4a.log 2>&1
