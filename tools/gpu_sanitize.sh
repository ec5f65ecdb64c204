# GPU: compute-sanitizer memcheck, racecheck and synccheck over tools/sanitize_cases.py
make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1
for T in memcheck racecheck synccheck; do
  X=""; [ $T = memcheck ] && X="--leak-check no"
  timeout 1500 compute-sanitizer --tool $T $X --error-exitcode 9 python tools/sanitize_cases.py > gpurun_out/sanitize_$T.log 2>&1; echo "rc=$?" >> gpurun_out/sanitize_$T.log
done
