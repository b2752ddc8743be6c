#!/bin/bash
# One gpurun call: ncu --set full (with source) of the fused kernel on one workload, plus the
# bench line of that workload.  Usage (GPU box, repo root): bash scripts/gpu_prof.sh TAG WORKLOAD [bench args]
TAG=$1; WL=$2; shift 2
OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 4 -c 1 \
    -o $OUT/prof_fused_$WL python bench.py --workload $WL --steps 2 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline "$@" > $OUT/ncu_full_$WL.log 2>&1
timeout 600 python bench.py --workload $WL --steps 20 --warmup 5 --no-cpu-baseline "$@" > $OUT/bench_$WL.json 2> $OUT/bench_$WL.err
