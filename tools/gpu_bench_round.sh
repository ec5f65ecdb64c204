# round-end style measurement: default bench line (C3, 40 trees, e2e, cpu_baseline), the reference
# arm, and the ncu launch list of one tree -> profiles/ncu_phases_<CFG>.json (traffic of the roofline)
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
CFG=${CFG:-C3}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
env $BENV timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/launches_$CFG.csv python bench.py --config $CFG --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch.log 2>&1
python tools/ncu_phases.py gpurun_out/launches_$CFG.csv $CFG ${DEPTH:-6} gpurun_out/ncu_phases_$CFG.json > /dev/null 2>&1
cp gpurun_out/ncu_phases_$CFG.json profiles/ 2>/dev/null
env $BENV timeout 900 python bench.py --config $CFG $BARGS > gpurun_out/bench_full_$CFG.log 2>&1
timeout 900 python bench.py --impl reference --config $CFG > gpurun_out/bench_ref_$CFG.log 2>&1
