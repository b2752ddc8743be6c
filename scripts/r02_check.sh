#!/bin/bash
# One gpurun call: GPU tests + short bench lines (C2, C3, C5) of the current build.
# Usage (GPU box): bash scripts/r02_check.sh TAG [pytest -k expr]
TAG=${1:-r02}; K=${2:-}
OUT=gpurun_out/$TAG; mkdir -p $OUT
python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; echo "smoke rc=$?" >> $OUT/smoke.log
if [ -n "$K" ]; then
  timeout 1500 python -m pytest tests -m gpu -q -k "$K" > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
else
  timeout 1500 python -m pytest tests -m gpu -q > $OUT/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.log
fi
for w in c2 c3 c5; do
  timeout 300 python bench.py --workload $w --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > $OUT/bench_$w.json 2> $OUT/bench_$w.err
done
tail -3 $OUT/pytest_gpu.log
