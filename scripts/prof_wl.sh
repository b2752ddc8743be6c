#!/bin/bash
# ncu --set full of the fused kernel on one workload (GPU box): bash scripts/prof_wl.sh TAG WL
TAG=$1; WL=$2; OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 3 -c 1 \
    -o $OUT/prof_fused_$WL python bench.py --workload $WL --steps 1 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline \
    > $OUT/ncu_$WL.log 2>&1
