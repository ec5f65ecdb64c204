nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt 2>&1
bash tools/gpu_all.sh
timeout 600 python bench.py > gpurun_out/bench_default.log 2>&1
