#!/bin/bash
# GPU box: time variant libraries on workloads.  Usage: bash scripts/tune_run.sh TAG "c2 c5" vbuild/libA.so vbuild/libB.so ...
TAG=$1; WLS=$2; shift 2
OUT=gpurun_out/$TAG; mkdir -p $OUT
for w in $WLS; do timeout 900 python scripts/tune_fused.py --workload $w "$@" >> $OUT/tune.jsonl 2>&1; done
cat $OUT/tune.jsonl | python -c "
import sys, json
for l in sys.stdin:
    try: d=json.loads(l); print(d.get('wl'), d['lib'].split('/')[-1], '%.4f ms'%d['ms'] if 'ms' in d else d.get('error','')[-300:])
    except Exception as e: print(l[:200])"
