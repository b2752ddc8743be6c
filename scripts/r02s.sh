OUT=gpurun_out/r02s; mkdir -p $OUT
START=$(date +%s)
timeout 1200 python bench.py > $OUT/bench_c4.json 2> $OUT/bench_c4.err
echo "bench wall $(( $(date +%s) - START )) s" >> $OUT/bench_c4.err
