#!/bin/bash
# ncu --set full of one kernel (regex $K, skip $S launches) of a short bench run of $CFG
CFG=${CFG:-C3}; K=${K:-k_sf_fast}; S=${S:-2}; TAG=${TAG:-x}
mkdir -p gpurun_out
ncu --set full --import-source on --clock-control none -k regex:$K -s $S -c 1 -o gpurun_out/${TAG}_${K}_$CFG -f \
    python bench.py --config $CFG --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > gpurun_out/ncu_${TAG}_${K}.log 2>&1
