#!/bin/bash
# One gpurun call for a round's evidence: smoke, GPU tests, bench lines of C1-C5 (+ C5 with the
# compact map domain, + the reference arm), ncu launch list (C2) and ncu --set full captures of
# the fused kernel on C2, C3 and C5, per-entry timings.  Usage (GPU box): bash scripts/round_check.sh TAG
TAG=${1:-r01}
bash scripts/gpu_check.sh $TAG c2
OUT=gpurun_out/$TAG
for w in c3 c5; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 4 -c 1 \
      -o $OUT/prof_fused_$w python bench.py --workload $w --steps 2 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline > $OUT/ncu_full_$w.log 2>&1
done
for w in c1 c3 c4 c5; do timeout 900 python bench.py --workload $w --steps 10 --warmup 3 > $OUT/bench_$w.json 2> $OUT/bench_$w.err; done
timeout 600 python bench.py --workload c5 --steps 10 --warmup 3 --no-cpu-baseline --reduce scatter > $OUT/bench_c5_compact.json 2> $OUT/bench_c5_compact.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > $OUT/bench_reference.json 2> $OUT/bench_reference.err
bash scripts/ops_check.sh $TAG "c2 c3"
