#!/bin/bash
# One gpurun call: build check, smoke, GPU parity tests, bench, ncu launch list + full capture.
# Usage (from the repo root, on the GPU box): bash scripts/gpu_check.sh [tag] [workload]
set -u
TAG=${1:-r01}
WL=${2:-c2}
OUT=gpurun_out/$TAG
mkdir -p $OUT
nvidia-smi > $OUT/nvidia-smi.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
timeout 600 python bench.py --workload $WL --steps 20 --warmup 5 > $OUT/bench.json 2> $OUT/bench.err; echo "bench rc=$?" >> $OUT/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches.csv \
    python bench.py --workload $WL --steps 3 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline > $OUT/ncu_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 4 -c 1 \
    -o ${REPDIR:-$OUT}/prof_fused python bench.py --workload $WL --steps 2 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline > $OUT/ncu_full.log 2>&1
echo done
