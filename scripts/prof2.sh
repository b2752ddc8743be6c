#!/bin/bash
# ncu --set full (with source) of the fused kernel on the given workloads.  Usage: bash scripts/prof2.sh TAG "c2 c5"
TAG=$1; WLS=${2:-c2}
OUT=gpurun_out/$TAG; mkdir -p $OUT
for w in $WLS; do
  timeout 600 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 4 -c 1 \
    -o $OUT/prof_$w python bench.py --workload $w --steps 2 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline > $OUT/ncu_$w.log 2>&1
done
