#!/bin/bash
# GPU box: measure the fp64 DFMA peak (burst + ~6 s sustained) with nvidia-smi clocks sampled
# during the run.  Writes gpurun_out/$TAG/fp64_peak.json and fp64_peak_clocks.csv.
# Usage: bash scripts/fp64_peak.sh TAG
TAG=${1:-r02}
OUT=gpurun_out/$TAG; mkdir -p $OUT
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/fp64_peak scripts/fp64_peak.cu || exit 1
nvidia-smi --query-gpu=timestamp,index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap \
    --format=csv -lms 200 > $OUT/fp64_peak_clocks.csv &
SMI=$!
sleep 0.5
/tmp/fp64_peak > $OUT/fp64_peak.json
RC=$?
sleep 0.3
kill $SMI
cat $OUT/fp64_peak.json
exit $RC
