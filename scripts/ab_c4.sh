# GPU box: A/B of library variants on C4 (bench.py, kernel time) and C2/C3/C5 (tune_fused).
# Usage: bash scripts/ab_c4.sh TAG lib1.so lib2.so ...
TAG=$1; shift; OUT=gpurun_out/$TAG; mkdir -p $OUT
export PYTHONPATH=.
for lib in "$@"; do
  TOASTB200_LIB=$(readlink -f $lib) timeout 600 python bench.py --workload c4 --steps 10 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/c4_$(basename $lib .so).json 2>/dev/null
  python -c "
import json; d=json.loads([l for l in open('$OUT/c4_$(basename $lib .so).json') if l.startswith('{')][-1]); print('c4', '$(basename $lib)', '%.3f ms'%d['roofline']['kernel_ms'], d['clocks']['reasons'])"
done
for w in c5 c2 c3; do timeout 900 python scripts/tune_fused.py --workload $w "$@" >> $OUT/tune.jsonl 2>&1; done
cat $OUT/tune.jsonl | python -c "
import sys, json
for l in sys.stdin:
    try: d=json.loads(l); print(d.get('wl'), d['lib'].split('/')[-1], '%.4f ms'%d['ms'] if 'ms' in d else d.get('error','')[-300:])
    except Exception as e: print(l[:200])"
