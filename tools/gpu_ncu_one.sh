# one --set full capture of kernel $K (launch index $S) on config $CFG; source page exported as CSV
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1
K=${K:-k_fused}; S=${S:-1}; CFG=${CFG:-C3}
timeout 600 ncu --set full --import-source on --clock-control none -k regex:$K -s $S -c 1 -o gpurun_out/full_${K}_$CFG -f \
  python bench.py --config $CFG --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_$K.log 2>&1
ncu -i gpurun_out/full_${K}_$CFG.ncu-rep --page source --csv --print-source sass > gpurun_out/src_${K}_$CFG.csv 2>&1
ncu -i gpurun_out/full_${K}_$CFG.ncu-rep --page source --csv --print-source cuda > gpurun_out/srccu_${K}_$CFG.csv 2>&1
