#!/bin/bash
# GPU box: A4 (build_noise_weighted) timing for library variants on C2/C3/C5.  Usage: bash scripts/a4_ab.sh TAG lib...
TAG=$1; shift; OUT=gpurun_out/$TAG; mkdir -p $OUT
export PYTHONPATH=.
for lib in "$@"; do
  for w in c2 c3 c5; do
    TOASTB200_LIB=$(readlink -f $lib) timeout 600 python scripts/bench_ops.py --workload $w --reps 10 --only "(A4)" 2>/dev/null \
      | python -c "
import sys, json
for l in sys.stdin:
    if l.startswith('{'):
        d = json.loads(l); print('$(basename $lib .so)', '$w', d['entry'], '%.4f ms' % d['ms'], d.get('hbm_frac'))"
  done
done | tee $OUT/a4.txt
