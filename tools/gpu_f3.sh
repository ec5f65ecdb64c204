make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
timeout 300 python -m pytest tests/test_gpu_variants.py -q -x > gpurun_out/variants_tests.log 2>&1; echo "rc=$?" >> gpurun_out/variants_tests.log
B="timeout 200 python bench.py --steps 20 --warmup 3 --no-e2e --no-cpu-baseline"
$B --config C5 --rle on --rle-split decompress > gpurun_out/abl_C5_rle_decompress.log 2>&1
