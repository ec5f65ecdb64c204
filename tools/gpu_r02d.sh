timeout 200 python -m pytest tests/test_gpu_parity.py -q -x -k fused > gpurun_out/fused_tests.log 2>&1; echo "rc=$?" >> gpurun_out/fused_tests.log
VARIANTS="s1c2 s2c2" CFGS="C3 C5" bash tools/gpu_variants.sh
