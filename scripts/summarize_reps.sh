#!/bin/bash
# GPU box: turn the round's .ncu-rep captures (kept outside gpurun_out/, which is size-capped) into
# text summaries + raw-page CSVs under gpurun_out/TAG.  Usage: bash scripts/summarize_reps.sh TAG REPDIR
TAG=$1; REPDIR=$2; OUT=gpurun_out/$TAG
ds() {  # det-samples per launch of workload $1, from its bench line
  python -c "
import json,sys
for f in ('$OUT/bench_$1.json', '$OUT/bench.json'):
    try:
        d = json.loads([l for l in open(f) if l.startswith('{')][-1])
        if d['config']['workload'].startswith('$1'): print(d['config']['det_samples_per_step']); sys.exit()
    except Exception: pass
print(0)"
}
for rep in $REPDIR/*.ncu-rep; do
  b=$(basename $rep .ncu-rep)
  case $b in
    prof_fused) w=c4 ;;
    prof_fused_*) w=${b#prof_fused_} ;;
    *) w=c2 ;;
  esac
  n=$(ds $w)
  extra=""
  [ "$b" = prof_fused ] && extra="--launches $OUT/launches.csv --bench $OUT/bench.json"
  python scripts/profile_summary.py --rep $rep --det-samples $n $extra --out $OUT/summary_$b.txt > /dev/null 2>&1
  ncu -i $rep --page raw --csv > $OUT/raw_$b.csv 2>/dev/null
done
ls -la $OUT > $OUT/listing.txt
