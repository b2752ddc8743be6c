OUT=gpurun_out/$1; mkdir -p $OUT
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pointing_to_map -s 3 -c 1 \
    -o $OUT/prof_c4 python bench.py --workload c4 --steps 1 --warmup 3 --soak 0 --no-e2e --no-cpu-baseline > $OUT/ncu_c4.log 2>&1
