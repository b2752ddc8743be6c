#!/bin/bash
# Time selected C-ABI entries for every library under build/variants (tuning aid, GPU box).
#   bash scripts/ops_variants.sh WORKLOAD ONLY OUT
WL=${1:-c2}; ONLY=${2:-}; OUT=${3:-gpurun_out/ops_variants.jsonl}
: > "$OUT"
for lib in build/variants/*.so; do
  echo "# $lib" >> "$OUT"
  TOASTB200_LIB=$lib python scripts/bench_ops.py --workload "$WL" --only "$ONLY" >> "$OUT" 2>&1
done
