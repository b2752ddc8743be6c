#!/bin/bash
# ncu --set full of the fused kernel for given library variants (tuning aid, GPU box).
# Usage: bash scripts/prof_variant.sh OUTDIR WORKLOAD lib1.so [lib2.so ...]
OUT=$1; WL=$2; shift 2
mkdir -p $OUT
for L in "$@"; do
  n=$(basename $L .so)
  TOASTB200_LIB=$(realpath $L) timeout 600 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 3 -c 1 \
     -o $OUT/$n python scripts/tune_fused.py --workload $WL > $OUT/$n.log 2>&1
done
