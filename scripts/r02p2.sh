#!/bin/bash
# GPU box: A/B of the pipelined predicated flush (PIPE) against the current kernel, plus fused parity
# tests on the PIPE build.  Usage: bash scripts/r02p2.sh TAG lib...
TAG=$1; shift; OUT=gpurun_out/$TAG; mkdir -p $OUT
export PYTHONPATH=.
bash scripts/ab_c4.sh $TAG "$@" > $OUT/ab.txt 2>&1
for lib in "$@"; do
  case $lib in *base*) continue;; esac
  TOASTB200_LIB=$(readlink -f $lib) timeout 900 python -m pytest tests/test_parity_gpu.py tests/test_parity_variants_gpu.py -x -q -m gpu -k "fused or round_trip" > $OUT/pytest_$(basename $lib .so).log 2>&1
  tail -2 $OUT/pytest_$(basename $lib .so).log >> $OUT/ab.txt
done
cat $OUT/ab.txt
