#!/bin/bash
# One gpurun call for a round's evidence: smoke, GPU tests, the default bench line (C4) with its
# ncu launch list and full capture, bench lines of every workload (+ C5 compact map domain,
# + C1 under a CUDA graph, + the reference arm), ncu --set full of the fused kernel on C2, C3, C5
# and of its scan mode (c3rt), per-entry timings.  Usage (GPU box): bash scripts/round_check.sh TAG
TAG=${1:-r02}
export PYTHONPATH=.
OUT=gpurun_out/$TAG
export REPDIR=/tmp/reps_$TAG; mkdir -p $REPDIR
bash scripts/gpu_check.sh $TAG c4
for w in c2 c3 c5 c3rt; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 4 -c 1 \
      -o $REPDIR/prof_fused_$w python bench.py --workload $w --steps 2 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline > $OUT/ncu_full_$w.log 2>&1
done
for w in c1 c2 c3 c5 c3rt c5m; do timeout 900 python bench.py --workload $w --steps 10 --warmup 3 > $OUT/bench_$w.json 2> $OUT/bench_$w.err; done
timeout 600 python bench.py --workload c1 --graph 10 --steps 50 --warmup 5 --no-cpu-baseline > $OUT/bench_c1_graph.json 2> $OUT/bench_c1_graph.err
timeout 600 python bench.py --workload c5 --steps 10 --warmup 3 --no-cpu-baseline --reduce scatter > $OUT/bench_c5_compact.json 2> $OUT/bench_c5_compact.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > $OUT/bench_reference.json 2> $OUT/bench_reference.err
bash scripts/ops_check.sh $TAG "c2 c3 c5"
REPDIR=$REPDIR bash scripts/prof_unfused.sh $TAG
bash scripts/summarize_reps.sh $TAG $REPDIR
