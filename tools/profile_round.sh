#!/bin/bash
# GPU side of the per-round profiles (run under gpurun from the repo root):
#   1. launch list of one C3 tree (cold-cache, serialised: shares, not absolute times)
#   2. ncu --set full of the streaming kernels, one launch each (level 2 of the first tree)
# Summaries are written here by tools/ncu_summary.py.
CFG=${CFG:-C3}
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
    -c 1500 --csv --log-file gpurun_out/launches_$CFG.csv \
    python bench.py --config $CFG --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_launch_$CFG.log 2>&1
for K in k_sf_fast k_part_scatter k_chunk_agg k_part_count; do
  ncu --set full --import-source on --clock-control none -k regex:$K -s 2 -c 1 -o gpurun_out/full_${K}_$CFG -f \
      python bench.py --config $CFG --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_full_${K}.log 2>&1
done
ls -la gpurun_out/
