#!/bin/bash
# One gpurun call: per-entry timings of every C-ABI entry (bench_ops.py) on several workloads,
# plus an ncu launch list with DRAM bytes per kernel for the C2 run.
# Usage (GPU box, repo root): bash scripts/ops_check.sh TAG "c2 c3 c5"
TAG=${1:-r01}; WLS=${2:-"c2 c3"}
OUT=gpurun_out/$TAG; mkdir -p $OUT
for wl in $WLS; do
  timeout 900 python scripts/bench_ops.py --workload $wl --reps 10 > $OUT/ops_$wl.jsonl 2> $OUT/ops_$wl.err
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  --csv --log-file $OUT/ops_ncu_c2.csv python scripts/bench_ops.py --workload c2 --reps 1 > $OUT/ops_ncu.log 2>&1
echo done
