#!/bin/bash
# Short bench lines of the fused kernel.  Usage (GPU box): bash scripts/quick_bench.sh TAG "c2 c3 c5" [extra bench args]
TAG=$1; WLS=${2:-"c2 c3 c5"}; shift 2
OUT=gpurun_out/$TAG; mkdir -p $OUT
for w in $WLS; do
  timeout 300 python bench.py --workload $w --steps 20 --warmup 3 --no-cpu-baseline --no-e2e "$@" > $OUT/bench_$w.json 2> $OUT/bench_$w.err
  python -c "
import json; d=json.loads(open('$OUT/bench_$w.json').read().strip().splitlines()[-1]); r=d['roofline']
print('$w', '%.3e'%d['value'], 'kern %.4f ms'%r['kernel_ms'], 'frac %.3f'%r['frac'])" 2>&1 | tail -1
done
