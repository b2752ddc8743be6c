#!/bin/bash
# GPU box: A4 / A5 timings for library variants on C2/C3/C5 + the unfused parity tests on each.
TAG=$1; shift; OUT=gpurun_out/$TAG; mkdir -p $OUT
export PYTHONPATH=.
for lib in "$@"; do
  for w in c2 c3 c5; do
    TOASTB200_LIB=$(readlink -f $lib) timeout 600 python scripts/bench_ops.py --workload $w --reps 10 --only "${ONLY:-(A4),(A5)}" 2>/dev/null \
      | python -c "
import sys, json
for l in sys.stdin:
    if l.startswith('{'):
        d = json.loads(l); print('$(basename $lib .so)', '$w', d['entry'], '%.4f ms' % d['ms'], d.get('hbm_frac'))"
  done
  TOASTB200_LIB=$(readlink -f $lib) timeout 900 python -m pytest tests/test_parity_gpu.py -x -q -m gpu -k "${KSEL:-noise_weighted or scan_map or round_trip}" 2>&1 | tail -1
done | tee $OUT/a5.txt
