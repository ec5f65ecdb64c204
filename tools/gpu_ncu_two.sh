# --set full captures of two kernels ($K1, $K2; launch index $S) on $CFG with env $BENV; SASS source pages
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1
CFG=${CFG:-C3}; S=${S:-1}
for K in $KS; do
env $BENV timeout 500 ncu --set full --import-source on --clock-control none -k regex:$K -s $S -c 1 -o gpurun_out/full_${K}_$CFG -f \
  python bench.py --config $CFG --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_$K.log 2>&1
ncu -i gpurun_out/full_${K}_$CFG.ncu-rep --page source --csv --print-source sass > gpurun_out/src_${K}_$CFG.csv 2>&1
done
