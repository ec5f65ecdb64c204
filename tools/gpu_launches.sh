# ncu launch list (durations + DRAM bytes) of one tree of $CFG; env $BENV applied
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1
CFG=${CFG:-C3}
env $BENV timeout 400 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none -c ${NC:-400} --csv \
  --log-file gpurun_out/launches_$CFG.csv python bench.py --config $CFG --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch.log 2>&1
